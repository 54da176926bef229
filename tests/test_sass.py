"""Static SASS guard (SURVEY §8a row a5, §8d "0 CALL/BRX for COAL/TP").

The paper's COAL / TypePointer keep the indirect call after resolution
(Table 1 row C; Fig. 5b line 4 `CALL R5`). This
build's grouped kernels replace it with a warp-grouped DIRECT, inlined call.
This test disassembles every kernel of the built libvf.so (cuobjdump, no GPU
needed) and asserts:
  * no register-operand CALL (indirect call) and no BRX (jump table) in ANY
    instantiation of the grouped dispatch kernels (k_dispatch_sorted /
    _grouped / _pipe), the fused step kernels (k_step_grouped), the
    persistent GOL run (k_run_grouped) and the ray tracer's direct kernel;
  * the config-2 (micro) grouped kernels contain no CALL at all (bodies
    fully inlined, no subroutine);
  * positive controls: the CUDA / SharedOA kernel (k_dispatch_virtual) and the
    paper-faithful indirect flavour (k_dispatch_indirect) DO contain register
    CALLs, so the scanner sees an indirect call when one is there.
"""
import concurrent.futures as cf
import glob
import os
import re
import shutil
import subprocess
import tempfile

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SO = os.path.join(ROOT, "paper_conf_asplos_zhangar21_b200", "libvf.so")
GROUPED = re.compile(r"\bvf::(k_dispatch_sorted|k_dispatch_grouped|k_dispatch_pipe|k_step_grouped"
                     r"|gol::k_run_grouped|gol::k_run_cluster_grouped|ray::k_ray_direct)\b")
INSN = re.compile(r"^\s+/\*[0-9a-f]+\*/\s+(?:@!?U?P[T0-9]+\s+)?(CALL|BRX|JMX)\S*\s+([^ ;,]+)")


def _sass(cubin):
    return subprocess.run(["cuobjdump", "-sass", cubin], capture_output=True, text=True, check=True).stdout


@pytest.fixture(scope="module")
def kernels():
    if not shutil.which("cuobjdump") or not shutil.which("c++filt"):
        pytest.skip("cuobjdump / c++filt not available")
    if not os.path.exists(SO):
        pytest.skip("libvf.so not built")
    stats = {}
    with tempfile.TemporaryDirectory() as td:
        subprocess.run(["cuobjdump", "-xelf", "all", SO], cwd=td, capture_output=True, check=True)
        cubins = sorted(glob.glob(os.path.join(td, "*.cubin")))
        assert cubins, "no sm_100a cubins in libvf.so"
        with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
            texts = list(ex.map(_sass, cubins))
    for text in texts:
        cur = None
        for line in text.splitlines():
            if "Function :" in line:
                cur = line.split("Function :", 1)[1].strip()
                stats[cur] = {"call_reg": 0, "call_imm": 0, "brx": 0}
                continue
            m = INSN.match(line)
            if m and cur:
                op, tgt = m.group(1), m.group(2)
                if op in ("BRX", "JMX"):
                    stats[cur]["brx"] += 1
                elif re.match(r"U?R\d+$", tgt):
                    stats[cur]["call_reg"] += 1
                else:
                    stats[cur]["call_imm"] += 1
    names = list(stats)
    dem = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True,
                         check=True).stdout.splitlines()
    return {d: stats[n] for n, d in zip(names, dem)}


def test_grouped_kernels_have_no_indirect_call_or_jump_table(kernels):
    grouped = {k: v for k, v in kernels.items() if GROUPED.search(k)}
    assert len(grouped) > 50, f"only {len(grouped)} grouped kernels found"
    bad = {k: v for k, v in grouped.items() if v["call_reg"] or v["brx"]}
    assert not bad, "indirect CALL / BRX in grouped kernels:\n" + "\n".join(f"{v} {k}" for k, v in bad.items())
    for app in ("micro::App", "gol::", "gen::", "graph::App", "traf::", "nbody::", "stut::", "collide::",
                "graph_en::VtxApp", "graph_en::EdgeApp", "ray::"):
        assert any(f"vf::{app}" in k for k in grouped), f"no grouped kernel of app {app}"


def test_micro_grouped_kernels_fully_inlined(kernels):
    micro = {k: v for k, v in kernels.items() if GROUPED.search(k) and "micro::App" in k}
    assert micro
    bad = {k: v for k, v in micro.items() if v["call_reg"] or v["call_imm"] or v["brx"]}
    assert not bad, "\n".join(f"{v} {k}" for k, v in bad.items())


def test_positive_controls_have_indirect_calls(kernels):
    virt = [v for k, v in kernels.items() if "vf::k_dispatch_virtual<vf::micro::App" in k]
    ind = [v for k, v in kernels.items() if "vf::k_dispatch_indirect<vf::micro::App" in k]
    assert virt and all(v["call_reg"] > 0 for v in virt)
    assert ind and all(v["call_reg"] > 0 for v in ind)
