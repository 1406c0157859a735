"""Literal layout pairs that exercise the stmatrix / ldmatrix instruction tiles
(Thm 5.1) — shared by the CPU (plan simulation, oracle bank model) and
GPU (parity) tests.  Literal basis tables only, no layout arithmetic.

Each entry: (name, spec_A, spec_B, elem_bytes, opts, expected (store, load) instruction
prefixes).  All run under faithful σ (the kernel holds the data exactly as A and B do)
with the SMEM exchange forced."""

OUT = [("i", 5), ("j", 5)]


def _s(reg, lane, warp):
    return {"out": OUT, "in": [("reg", reg), ("lane", lane), ("warp", warp)]}


MATRIX_CASES = [
    # stmatrix.x1 (one word register) -> ldmatrix.x1.trans: the row {j0,j1,j2} is
    # (word, lane 0, lane 1) of A and lanes 2-4 of B
    ("x1_mat_to_trans_b16",
     _s(["j0"], ["j1", "j2", "i0", "i1", "i2"], ["j3", "j4", "i3", "i4"]),
     _s(["i0"], ["i1", "i2", "j0", "j1", "j2"], ["j3", "j4", "i3", "i4"]), 2,
     ("stmatrix.m8n8.x1.b16", "ldmatrix.m8n8.x1.trans.b16")),
    # 4-byte elements: k = 0, the row is lanes 0,1 on both sides; one select bit -> .x2
    ("x2_mat_mat_b32",
     _s(["i4"], ["j0", "j1", "i0", "i1", "i2"], ["j2", "j3", "j4", "i3"]),
     _s(["i3"], ["j0", "j1", "i2", "i1", "i0"], ["j2", "j3", "j4", "i4"]), 4,
     ("stmatrix.m8n8.x2.b16", "ldmatrix.m8n8.x2.b16")),
    # 1-byte elements: two word bits, lanes 0,1 -> a 16-byte row; vectorised loads
    ("x4_mat_to_vec_b8",
     _s(["j0", "j1", "i0", "i1"], ["j2", "j3", "i2", "i3", "i4"], ["j4"]),
     _s(["j0", "j1", "j2", "j3"], ["i0", "i1", "i2", "i3", "i4"], ["j4"]), 1,
     ("stmatrix.m8n8.x4.b16", "ld.shared.v4.b32")),
    # transposed stores: A's lanes 2-4 are the row B holds in registers
    ("x4_trans_to_vec_b16",
     _s(["i0", "i3", "i4"], ["i1", "i2", "j0", "j1", "j2"], ["j3", "j4"]),
     _s(["j0", "j1", "j2"], ["i0", "i1", "i2", "i3", "i4"], ["j3", "j4"]), 2,
     ("stmatrix.m8n8.x4.trans.b16", "ld.shared.v4.b32")),
]
