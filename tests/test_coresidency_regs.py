"""The GEMM-concurrent swap kernels must co-reside with a cuBLAS GEMM CTA
(DESIGN.md §7c): its 8 warps x 168 registers leave 5632 registers in each of
an SM's four 16K-register sub-partitions, so every warp of bulk shapes 7 and
9 and of the capped direct shape 9 must stay at <= 176 registers per thread
(a bulk-9 build at 180 lost co-residency and cost the GEMM +80%,
profiles/r02/hybrid/pace_180regs_gemm.jsonl).  Checked from the ptxas report
the build writes (build/swap_kernels.cu.ptxas.txt); no GPU needed."""
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PTXAS = os.path.join(ROOT, "build", "swap_kernels.cu.ptxas.txt")

# mangled template arguments of the kernels that run beside a GEMM
GEMM_SIDE = {
    "bulk 7": re.compile(r"mp_swap_bulk(_g)?ILi\dELi12ELi4ELi\d+ELi0E"),
    "bulk 9": re.compile(r"mp_swap_bulk(_g)?ILi\dELi12ELi4ELi\d+ELi1E"),
    "direct 9": re.compile(r"mp_swap_direct(_g)?ILi\dELi128ELi8ELi32ELb0ELb1ELi\d+E"),
}


def _registers():
    out, cur = {}, None
    for line in open(PTXAS):
        m = re.search(r"Compiling entry function '(\S+)'", line)
        if m:
            cur = m.group(1)
            continue
        m = re.search(r"Used (\d+) registers", line)
        if m and cur:
            out[cur] = int(m.group(1))
            cur = None
    return out


@pytest.mark.skipif(not os.path.exists(PTXAS), reason="build/ not present (run __graft_entry__.build())")
def test_gemm_side_kernels_fit_beside_a_gemm_cta():
    regs = _registers()
    for name, pat in GEMM_SIDE.items():
        found = {k: v for k, v in regs.items() if pat.search(k)}
        assert found, "no %s kernel in the ptxas report" % name
        worst = max(found.values())
        assert worst <= 176, "%s uses %d registers per thread (> 176: no co-residency with a GEMM CTA)" % (name, worst)
