"""Program tables ("virtual SASS") — transcribed from docs/EVENT_MODEL.md §3.

A program is a dict of equal-length numpy arrays indexed by pc:
opcode, kind, width, bb, is_leader, guarded; plus n_opcodes and n_bbs.
The BB rule (P:L115–117 (§4), reading R-14) is checked by tests/test_oracle_programs.py.
"""
from __future__ import annotations

import numpy as np

from .mix import R

ALU, CTRL, GLD, GST, GATOM, OTHERMEM = range(6)
MEM_KINDS = (GLD, GST, GATOM)

S2R, IMAD, ISETP, EXIT, IMAD_WIDE, LDG, STG, FADD, FFMA, MOV, IADD, BRA, SEL = range(13)
N_OPCODES_WL = 16
# §3.6 (F4) opcode ids
SHFL, FMUL, LOP3, I2F, MUFU_SIN, MUFU_COS, FSEL, BREV, SHF, WFFT32 = range(13, 23)
N_OPCODES_WFFT = 32


def _table(rows, n_opcodes=N_OPCODES_WL):
    """rows: (opcode, kind, width, bb, is_leader, guarded[, branch_target])."""
    cols = list(zip(*[r[:6] for r in rows]))
    prog = {
        "opcode": np.array(cols[0], dtype=np.int64),
        "kind": np.array(cols[1], dtype=np.int64),
        "width": np.array(cols[2], dtype=np.int64),
        "bb": np.array(cols[3], dtype=np.int64),
        "is_leader": np.array(cols[4], dtype=np.int64),
        "guarded": np.array(cols[5], dtype=np.int64),
        "target": np.array([r[6] if len(r) > 6 else -1 for r in rows], dtype=np.int64),
    }
    prog["n_pcs"] = len(rows)
    prog["n_opcodes"] = n_opcodes
    prog["n_bbs"] = int(prog["bb"].max()) + 1
    return prog


def vectoradd():
    """§3.1, 13 pcs, 2 BBs."""
    return _table([
        (S2R, ALU, 0, 0, 1, 0), (S2R, ALU, 0, 0, 0, 0), (IMAD, ALU, 0, 0, 0, 0), (ISETP, ALU, 0, 0, 0, 0),
        (EXIT, CTRL, 0, 0, 0, 1),
        (IMAD_WIDE, ALU, 0, 1, 1, 0), (IMAD_WIDE, ALU, 0, 1, 0, 0), (LDG, GLD, 4, 1, 0, 0), (LDG, GLD, 4, 1, 0, 0),
        (IMAD_WIDE, ALU, 0, 1, 0, 0), (FADD, ALU, 0, 1, 0, 0), (STG, GST, 4, 1, 0, 0), (EXIT, CTRL, 0, 1, 0, 0),
    ])


def sgemm():
    """§3.2, 18 pcs, 4 BBs."""
    return _table([
        (S2R, ALU, 0, 0, 1, 0), (S2R, ALU, 0, 0, 0, 0), (S2R, ALU, 0, 0, 0, 0), (S2R, ALU, 0, 0, 0, 0),
        (IMAD, ALU, 0, 0, 0, 0), (IMAD, ALU, 0, 0, 0, 0), (ISETP, ALU, 0, 0, 0, 0), (EXIT, CTRL, 0, 0, 0, 1),
        (MOV, ALU, 0, 1, 1, 0), (MOV, ALU, 0, 1, 0, 0),
        (LDG, GLD, 4, 2, 1, 0), (LDG, GLD, 4, 2, 0, 0), (FFMA, ALU, 0, 2, 0, 0), (IADD, ALU, 0, 2, 0, 0),
        (ISETP, ALU, 0, 2, 0, 0), (BRA, CTRL, 0, 2, 0, 1, 10),
        (STG, GST, 4, 3, 1, 0), (EXIT, CTRL, 0, 3, 0, 0),
    ])


def bfs():
    """§3.3, 36 pcs over two kernels, 11 BBs."""
    return _table([
        # kernel 1
        (S2R, ALU, 0, 0, 1, 0), (S2R, ALU, 0, 0, 0, 0), (IMAD, ALU, 0, 0, 0, 0), (ISETP, ALU, 0, 0, 0, 0),
        (EXIT, CTRL, 0, 0, 0, 1),
        (LDG, GLD, 1, 1, 1, 0), (ISETP, ALU, 0, 1, 0, 0), (BRA, CTRL, 0, 1, 0, 1, 21),
        (STG, GST, 1, 2, 1, 0), (LDG, GLD, 4, 2, 0, 0), (LDG, GLD, 4, 2, 0, 0), (ISETP, ALU, 0, 2, 0, 0),
        (BRA, CTRL, 0, 2, 0, 1, 21),
        (LDG, GLD, 4, 3, 1, 0), (LDG, GLD, 1, 3, 0, 0), (ISETP, ALU, 0, 3, 0, 0), (BRA, CTRL, 0, 3, 0, 1, 18),
        (STG, GST, 1, 4, 1, 0),
        (IADD, ALU, 0, 5, 1, 0), (ISETP, ALU, 0, 5, 0, 0), (BRA, CTRL, 0, 5, 0, 1, 13),
        (EXIT, CTRL, 0, 6, 1, 0),
        # kernel 2
        (S2R, ALU, 0, 7, 1, 0), (S2R, ALU, 0, 7, 0, 0), (IMAD, ALU, 0, 7, 0, 0), (ISETP, ALU, 0, 7, 0, 0),
        (EXIT, CTRL, 0, 7, 0, 1),
        (LDG, GLD, 1, 8, 1, 0), (ISETP, ALU, 0, 8, 0, 0), (BRA, CTRL, 0, 8, 0, 1, 35),
        (STG, GST, 1, 9, 1, 0), (STG, GST, 1, 9, 0, 0), (STG, GST, 4, 9, 0, 0), (STG, GST, 1, 9, 0, 0),
        (STG, GST, 4, 9, 0, 0),
        (EXIT, CTRL, 0, 10, 1, 0),
    ])


def stencil():
    """§3.4, 21 pcs, 2 BBs."""
    return _table([
        (S2R, ALU, 0, 0, 1, 0), (S2R, ALU, 0, 0, 0, 0), (S2R, ALU, 0, 0, 0, 0), (S2R, ALU, 0, 0, 0, 0),
        (IMAD, ALU, 0, 0, 0, 0), (IMAD, ALU, 0, 0, 0, 0), (ISETP, ALU, 0, 0, 0, 0), (EXIT, CTRL, 0, 0, 0, 1),
        (ISETP, ALU, 0, 1, 1, 0), (LDG, GLD, 4, 1, 0, 0),
        (LDG, GLD, 4, 1, 0, 1), (LDG, GLD, 4, 1, 0, 1), (LDG, GLD, 4, 1, 0, 1), (LDG, GLD, 4, 1, 0, 1),
        (FADD, ALU, 0, 1, 0, 1), (FADD, ALU, 0, 1, 0, 1), (FADD, ALU, 0, 1, 0, 1), (FFMA, ALU, 0, 1, 0, 1),
        (SEL, ALU, 0, 1, 0, 0), (STG, GST, 4, 1, 0, 0), (EXIT, CTRL, 0, 1, 0, 0),
    ])


def wfft_emu():
    """§3.6 program WFFT_EMU (Listing 10 analogue): 14 pcs, 3 BBs."""
    return _table([
        (S2R, ALU, 0, 0, 1, 0), (S2R, ALU, 0, 0, 0, 0), (IMAD, ALU, 0, 0, 0, 0), (ISETP, ALU, 0, 0, 0, 0),
        (EXIT, CTRL, 0, 0, 0, 1),
        (IMAD_WIDE, ALU, 0, 1, 1, 0), (LDG, GLD, 8, 1, 0, 0), (WFFT32, ALU, 0, 1, 0, 0),
        (IMAD_WIDE, ALU, 0, 1, 0, 0), (STG, GST, 8, 1, 0, 0), (IADD, ALU, 0, 1, 0, 0), (ISETP, ALU, 0, 1, 0, 0),
        (BRA, CTRL, 0, 1, 0, 1, 5),
        (EXIT, CTRL, 0, 2, 1, 0),
    ], n_opcodes=N_OPCODES_WFFT)


def wfft_sw():
    """§3.6 program WFFT_SW (the transform written in CUDA): 83 pcs, 4 BBs."""
    rows = [(S2R, ALU, 0, 0, 1, 0), (S2R, ALU, 0, 0, 0, 0), (IMAD, ALU, 0, 0, 0, 0), (ISETP, ALU, 0, 0, 0, 0),
            (EXIT, CTRL, 0, 0, 0, 1)]
    for q in range(4):                                   # twiddle setup, pcs 5-36
        for o in (LOP3, LOP3, ISETP, I2F, MUFU_SIN, MUFU_COS, FSEL, FSEL):
            rows.append((o, ALU, 0, 1, 1 if len(rows) == 5 else 0, 0))
    rows += [(BREV, ALU, 0, 1, 0, 0), (SHF, ALU, 0, 1, 0, 0)]
    rows += [(IMAD_WIDE, ALU, 0, 2, 1, 0), (LDG, GLD, 8, 2, 0, 0)]   # pcs 39, 40
    for q in range(4):                                   # stages h = 16, 8, 4, 2: pcs 41-72
        for o in (SHFL, SHFL, FFMA, FFMA, FMUL, FFMA, FMUL, FFMA):
            rows.append((o, ALU, 0, 2, 0, 0))
    for o in (SHFL, SHFL, FFMA, FFMA):                   # stage h = 1: pcs 73-76
        rows.append((o, ALU, 0, 2, 0, 0))
    rows += [(IMAD_WIDE, ALU, 0, 2, 0, 0), (STG, GST, 8, 2, 0, 0), (IADD, ALU, 0, 2, 0, 0),
             (ISETP, ALU, 0, 2, 0, 0), (BRA, CTRL, 0, 2, 0, 1, 39), (EXIT, CTRL, 0, 3, 1, 0)]
    assert len(rows) == 83
    return _table(rows, n_opcodes=N_OPCODES_WFFT)


def replay():
    """§3.5: 4096 pcs, 64 opcodes, 512 BBs, generated from h = R(pc, 100) with the constant SEED."""
    from .mix import SEED
    seed = SEED
    pc = np.arange(4096, dtype=np.uint64)
    h = R(pc, 100, seed)
    mem = (h % np.uint64(4)) == 0
    st = ((h >> np.uint64(8)) & np.uint64(1)) == 1
    kind = np.where(mem, np.where(st, GST, GLD), np.where((pc & np.uint64(7)) == 7, CTRL, ALU))
    width = np.where(mem, 4 << ((h >> np.uint64(16)) % np.uint64(3)).astype(np.int64), 0)
    opcode = np.where(mem, np.where(kind == GLD, 0, 1), 2 + ((h >> np.uint64(24)) % np.uint64(62)).astype(np.int64))
    pcs = np.arange(4096, dtype=np.int64)
    prog = {
        "opcode": opcode.astype(np.int64),
        "kind": kind.astype(np.int64),
        "width": width.astype(np.int64),
        "bb": pcs >> 3,
        "is_leader": ((pcs & 7) == 0).astype(np.int64),
        "guarded": np.ones(4096, dtype=np.int64),
        "target": -np.ones(4096, dtype=np.int64),
        "n_pcs": 4096,
        "n_opcodes": 64,
        "n_bbs": 512,
    }
    return prog


def is_mem(prog):
    return np.isin(prog["kind"], MEM_KINDS)
