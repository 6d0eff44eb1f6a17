"""compute-sanitizer runs over small instances of every template:
memcheck (out-of-bounds / misaligned accesses), racecheck (shared-memory hazards) and
synccheck (barrier misuse).  One process per tool runs all cases of tools/sanitize_cases.py."""
import os
import shutil
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool):
    cs = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    if not os.path.exists(cs):
        pytest.skip("compute-sanitizer not installed")
    if os.environ.get("MDH_SANITIZER") != "1":
        # the GPU pool refuses compute-sanitizer (runs under it have left GPUs needing a
        # reset); opt in with MDH_SANITIZER=1 on a box that allows it
        pytest.skip("compute-sanitizer runs are opt-in (MDH_SANITIZER=1)")
    cmd = [cs, "--tool", tool, "--error-exitcode", "9", "--target-processes", "all",
           sys.executable, os.path.join(ROOT, "tools", "sanitize_cases.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1500, cwd=ROOT)
    out = r.stdout + r.stderr
    if "closed on this pool" in out:
        pytest.skip("compute-sanitizer is closed on this GPU pool")
    if tool == "racecheck":
        # The only accepted report: the 2-SM kernel's `tcgen05.alloc.cta_group::2`, where both
        # CTAs of the pair allocate and the hardware writes the (identical) TMEM address into
        # the slot — both accesses are attributed to the alloc line itself.
        src = open(os.path.join(ROOT, "paper_conf_sc_schulzegr25_b200", "csrc", "t4_tcgen05.cu")).read().splitlines()
        alloc = [i + 1 for i, l in enumerate(src) if "tcgen05.alloc.cta_group::2" in l]
        assert alloc, "alloc line not found"
        ok_lines = {f"t4_tcgen05.cu:{a + d}" for a in alloc for d in (0, 1)}   # the asm spans 2 lines
        for blk in out.split("Race reported")[1:]:
            blk = blk.split("SUMMARY")[0]
            located = [l for l in blk.splitlines() if "access at" in l and " in " in l]
            assert located and all(any(k in l for k in ok_lines) for l in located), blk[:800]
            assert "gemm2_kernel" in blk, blk[:800]
        assert "ok" in out and "Traceback" not in out, out[-4000:]
        return
    assert r.returncode == 0, out[-4000:]
    assert "ERROR SUMMARY: 0 errors" in out, out[-4000:]
