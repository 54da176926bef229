#!/usr/bin/env python
"""Config-3 launch-shape sweep: shape parts (vf_set_tuning "ray_parts") x rays
per thread ("ray_rays") for the direct COAL / TypePointer ray kernel at
1920x1080 x 10,000 shapes. One JSON line per point; frames are checked equal
to the first point's (hit ids and RGB, bit for bit).

    python tools/sweep_ray.py --parts -1,1,3,5,7,8 --rays 4 --variants typeptr,coal
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import torch  # noqa: E402

import synth  # noqa: E402
from apps_bench import Env  # noqa: E402
from paper_conf_asplos_zhangar21_b200 import vf  # noqa: E402
from paper_conf_asplos_zhangar21_b200.ray import Ray  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--parts", default="-1,1,3,5,7,8")
    ap.add_argument("--rays", default="4")
    ap.add_argument("--variants", default="typeptr,coal")
    ap.add_argument("--steps", type=int, default=10)
    a = ap.parse_args()
    W, H, S = 1920, 1080, 10000
    ctx = vf.Ctx(0)
    env = Env(ctx)
    types, P = synth.ray_scene(S, seed=7)
    cam = synth.ray_camera(W, H)
    ref = None
    for v in a.variants.split(","):
        r = Ray(ctx, types, P, v)
        for nr in [int(x) for x in a.rays.split(",")]:
            for parts in [int(x) for x in a.parts.split(",")]:
                vf.set_tuning("ray_rays", nr)
                vf.set_tuning("ray_parts", parts)
                out = {}

                def step():
                    out["f"] = r.render(W, H, cam)
                ms = env.timed(step, a.steps, 2)
                rgb, hid = out["f"]
                ok = True
                if ref is None:
                    ref = (rgb.clone(), hid.clone())
                else:
                    ok = bool(torch.equal(ref[0], rgb) and torch.equal(ref[1], hid))
                print(json.dumps({"variant": v, "rays": nr, "parts": parts, "ms_per_frame": ms,
                                  "gcalls_per_s": W * H * S / (ms / 1e3) / 1e9, "agree": ok}), flush=True)
        del r
        env.free()
    vf.set_tuning("ray_parts", -1)
    vf.set_tuning("ray_rays", 4)
    ctx.close()


if __name__ == "__main__":
    main()
