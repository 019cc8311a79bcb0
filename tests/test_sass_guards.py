"""SASS-level guards (no GPU): the compiled liblime.so must contain the instructions the design
relies on. cuobjdump runs on the CPU box."""
import re
import shutil
import subprocess

import pytest

from paper_conf_pldi_dubachcrbf12_b200 import build as lime_build

pytestmark = pytest.mark.skipif(shutil.which("cuobjdump") is None, reason="cuobjdump not available")


@pytest.fixture(scope="module")
def sass():
    lib = lime_build.build()
    out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True, check=True).stdout
    funcs, cur = {}, None
    for line in out.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            cur = m.group(1)
            funcs[cur] = []
        elif cur and re.match(r"\s+/\*[0-9a-f]{4}\*/", line):
            funcs[cur].append(re.sub(r"^\s+/\*[0-9a-f]+\*/\s+", "", line).split(";")[0])
    return funcs


def _fn(sass, pat):
    hits = [k for k in sass if re.search(pat, k)]
    assert hits, pat
    return [i for k in hits for i in sass[k]]


def test_mandelbrot_has_no_inexact_fma(sass):
    # R7 bit-exactness: every FFMA/FFMA2 in the Mandelbrot kernel must be an exact rewrite of
    # R7's ops (multiplier +-1 immediate: one add/sub; multiplier 2: (a + a) + c, where a + a is
    # exact so R7's two roundings equal the fma's one), never a contracted x*y+z.
    for ins in _fn(sass, r"mandel"):
        if re.match(r"(@!?P\d )?FFMA", ins):
            assert re.search(r",\s*(-?1|2)(\.0+)?\s*,", ins), ins


def test_mandelbrot_uses_packed_fp32(sass):
    ops = " ".join(_fn(sass, r"mandel"))
    assert "FMUL2" in ops and "FADD2" in ops


def test_nbody_uses_packed_fp32_and_mufu_and_bulk_copy(sass):
    ops = " ".join(_fn(sass, r"force_kernelILi256ELi4ELb1"))
    assert "FFMA2" in ops and "MUFU.RSQ" in ops
    assert "UBLKCP" in ops                         # cp.async.bulk (1-D TMA) staging of j-tiles
    assert "LDS.128" in ops                        # broadcast reads of the staged sources


def test_gemm_is_tcgen05(sass):
    for pat in (r"gemm_kernel", r"gemm2_kernel", r"gemm_wide_kernel"):
        ops = " ".join(_fn(sass, pat))
        assert "UTCHMMA" in ops or "UTCQMMA" in ops   # tcgen05.mma
        assert "UTMALDG" in ops                        # TMA tensor loads
        assert "LDTM" in ops                           # tcgen05.ld epilogue
        assert "HMMA" not in ops.replace("UTCHMMA", "")


@pytest.mark.parametrize("kernel", [r"gemm2_kernel", r"gemm_wide_kernel"])
def test_pair_gemms_are_two_cta_tcgen05_with_tma_store(sass, kernel):
    # the production kernels (gemm_wide_kernel is the default for M >= 256,
    # N >= 512 since round 2): cta_group::2 MMAs, pair-wide TMA loads, TMA-store epilogue, tcgen05.ld
    ops = " ".join(_fn(sass, kernel))
    assert "UTCHMMA.2CTA" in ops
    assert "UTMALDG" in ops
    assert "UTMASTG" in ops
    assert "LDTM" in ops


def test_idea_loop_instruction_count_matches_bench(sass):
    # bench.py's JG-Crypt issue roofline divides by IDEA_SASS_PER_UNIT: the grid-stride loop body
    # (one 16-byte unit = two IDEA blocks) must still be that long (+-3 %)
    import re
    import bench
    lib = lime_build.build()
    out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True, check=True).stdout
    lines, cur = [], False
    for line in out.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            cur = "idea_kernel" in m.group(1)
        elif cur:
            lines.append(line)
    addr = [int(m.group(1), 16) for ln in lines for m in [re.search(r"/\*([0-9a-f]{4})\*/", ln)] if m]
    back = [(int(m.group(2), 16), int(m.group(1), 16)) for ln in lines
            for m in [re.search(r"/\*([0-9a-f]{4})\*/\s+@!?P\d\s+BRA\s+0x([0-9a-f]+)", ln)] if m]
    loops = [(dst, src) for dst, src in back if dst < src]
    assert loops and addr
    dst, src = max(loops, key=lambda x: x[1] - x[0])
    n = (src - dst) // 16 + 1
    assert abs(n - bench.IDEA_SASS_PER_UNIT) <= 0.03 * bench.IDEA_SASS_PER_UNIT, n
