"""C-ABI library checks that need no GPU: it loads, exports every symbol include/*.h declares, and its
host-only entry points behave (program tables, sizes, argument validation, host digest)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_micro_villasnk19_b200", "libnvbt.so")
pytestmark = pytest.mark.skipif(not os.path.exists(LIB), reason="libnvbt.so not built")


def declared_symbols():
    names = set()
    for h in ("nvbt.h", "nvbt_workloads.h"):
        txt = open(os.path.join(ROOT, "include", h)).read()
        txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
        names |= set(re.findall(r"\b(nvbt_[a-z0-9_]+)\s*\(", txt))
    return names - {"nvbt_drain_fn"}


def test_every_declared_symbol_is_exported():
    lib = C.CDLL(LIB)
    names = declared_symbols()
    assert len(names) >= 25
    missing = [n for n in sorted(names) if not hasattr(lib, n)]
    assert missing == []


def test_binding_covers_declared_symbols():
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    assert declared_symbols() <= set(nb.EXPORTED)
    assert nb.nvbt_abi_version() == 1


@pytest.mark.parametrize("w,name", [(1, "vectoradd"), (2, "sgemm"), (3, "bfs"), (4, "stencil"), (5, "replay"),
                                    (6, "wfft_emu"), (7, "wfft_sw")])
def test_program_tables_match_oracle_transcription(w, name):
    """Both sides transcribe docs/EVENT_MODEL.md §3 independently; the tables must agree."""
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    from oracle import programs
    arr, n_ops, n_bbs = nb.nvbt_program(w)
    got = nb.program_numpy(arr)
    exp = getattr(programs, name)()
    assert n_ops == exp["n_opcodes"] and n_bbs == exp["n_bbs"] and len(arr) == exp["n_pcs"]
    for k in got:
        assert (got[k] == exp[k]).all(), k


def test_workspace_and_validation_errors():
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    assert nb.nvbt_workspace_size(18, 16, 4, nb.COUNT) > 0
    big = nb.nvbt_workspace_size(18, 16, 4, nb.COUNT | nb.PER_WARP, n_warps=1 << 20)
    assert big >= 16 * (1 << 20)
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_workspace_size(0, 16, 4, nb.COUNT)
    assert e.value.code == nb.EINVAL
    with pytest.raises(nb.NvbtError):
        nb.nvbt_workspace_size(18, 16, 4, nb.PER_WARP)   # PER_WARP needs n_warps
    with pytest.raises(nb.NvbtError):
        nb.nvbt_workspace_size(18, 16, 4, 1 << 9)        # unknown flag
    assert nb.nvbt_workload_warps(nb.W_SGEMM, 1024, 1024) == 32768
    assert nb.nvbt_workload_warps(nb.W_VECTORADD, 65500) == 2048
    assert nb.nvbt_workload_warps(nb.W_STENCIL, 8192) == 2097152


def test_host_digest_matches_oracle():
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    from oracle import events as ev, programs, trace
    from oracle.models import stencil
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    stencil.run(acc, 64, 1 << 32, (1 << 32) + (1 << 24))
    recs = acc.record_array()
    assert nb.nvbt_digest_records(recs) == (acc.digest.n, acc.digest.d1, acc.digest.d2)


def _encode_compact(recs, wide_mask):
    """Test-side encoder of EM §5.1 (written from the spec): record r -> one compact slot, or a wide pair
    when wide_mask[r]."""
    import struct
    out = []
    for r, rec in enumerate(recs):
        b = bytes(rec)
        A, P = struct.unpack_from("<II", b, 16)
        E = A & P
        addr = struct.unpack_from("<32Q", b, 32)
        kind = b[27]
        if not wide_mask[r]:
            lanes = [l for l in range(32) if (E >> l) & 1]
            base = addr[lanes[0]]
            sl = bytearray(176)
            sl[0:27] = b[0:27]
            sl[27] = kind | 0x80
            struct.pack_into("<Q", sl, 32, base)
            for l in lanes:
                struct.pack_into("<i", sl, 48 + 4 * l, addr[l] - base)
            out.append(sl)
        else:
            for h, flag in ((0, 0x40), (1, 0x20)):
                sl = bytearray(176)
                sl[0:27] = b[0:27]
                sl[27] = kind | flag
                sl[32:160] = b[32 + 128 * h:160 + 128 * h]
                out.append(sl)
    return np.frombuffer(b"".join(out), dtype=np.uint8).reshape(-1, 176)


def test_compact_decode_matches_records():
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    from oracle import events as ev, programs
    from oracle.models import stencil
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    stencil.run(acc, 64, 1 << 32, (1 << 32) + (1 << 24))
    recs = acc.record_array()
    wide = np.random.default_rng(0).random(len(recs)) < 0.3
    slots = _encode_compact(recs, wide)
    assert len(slots) == len(recs) + wide.sum()
    dec = nb.nvbt_decode_compact(slots)
    assert dec.shape == recs.shape and (dec == recs).all()
    with pytest.raises(nb.NvbtError):          # an unpaired wide half is rejected
        nb.nvbt_decode_compact(slots[(slots[:, 27] & 0xE0) == 0x20][:1])
    with_skips = _with_skip_slots(slots, 176, seed=3)
    assert len(with_skips) > len(slots)
    assert np.array_equal(nb.nvbt_decode_compact(with_skips), dec)


def _with_skip_slots(slots, width, seed):
    """Inserts 0-2 skip slots (0xC0 at byte 27, other bytes random: unused tickets of a producer's block)
    after every record of a packed slot array; never inside a multi-slot record."""
    rng = np.random.default_rng(seed)
    starts = [i for i in range(len(slots)) if (slots[i, 27] & 0xE0) != 0x20]
    pieces = []
    for k, i in enumerate(starts):
        j = starts[k + 1] if k + 1 < len(starts) else len(slots)
        pieces.append(slots[i:j])
        for _ in range(int(rng.integers(0, 3))):
            junk = rng.integers(0, 256, size=(1, width), dtype=np.uint8)
            junk[0, 27] = 0xC0 | (junk[0, 27] & 0x1F)
            pieces.append(junk)
    return np.concatenate(pieces)


def _encode_compact128(recs, long_mask):
    """Test-side encoder of EM §5.2 (written from the spec): record r -> one 128 B short slot (base + 32 x
    i16 deltas), or three slots of full addresses when long_mask[r] (or a delta does not fit 16 bits)."""
    import struct
    out = []
    for r, rec in enumerate(recs):
        b = bytes(rec)
        A, P = struct.unpack_from("<II", b, 16)
        E = A & P
        addr = struct.unpack_from("<32Q", b, 32)
        kind = b[27]
        lanes = [l for l in range(32) if (E >> l) & 1]
        base = addr[lanes[0]]
        fits = all(-32768 <= addr[l] - base <= 32767 for l in lanes)
        if fits and not long_mask[r]:
            sl = bytearray(128)
            sl[0:27] = b[0:27]
            sl[27] = kind | 0x80
            struct.pack_into("<Q", sl, 32, base)
            for l in lanes:
                struct.pack_into("<h", sl, 40 + 2 * l, addr[l] - base)
            out.append(sl)
        else:
            s0 = bytearray(128)
            s0[0:27] = b[0:27]
            s0[27] = kind | 0x40
            struct.pack_into("<12Q", s0, 32, *addr[0:12])
            s1, s2 = bytearray(128), bytearray(128)
            for sl, lo in ((s1, 12), (s2, 27)):
                sl[27] = 0x20
                struct.pack_into("<3Q", sl, 0, *addr[lo:lo + 3])
                rest = addr[lo + 3:min(lo + 15, 32)]
                struct.pack_into(f"<{len(rest)}Q", sl, 32, *rest)
            out += [s0, s1, s2]
    return np.frombuffer(b"".join(out), dtype=np.uint8).reshape(-1, 128)


def test_compact128_decode_matches_records():
    """EM §5.2 slots decode back to the EM §5 records (stencil records as short slots, 30 % forced long, and
    BFS-like records whose spans need the long form)."""
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    from oracle import events as ev, programs
    from oracle.models import stencil
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    stencil.run(acc, 64, 1 << 32, (1 << 32) + (1 << 24))
    recs = acc.record_array().copy()
    words = recs.view("<u8").reshape(-1, 36)
    hdr = recs.view("<u4").reshape(-1, 72)
    lane5 = ((hdr[:, 4] & hdr[:, 5]) >> 5) & 1 == 1          # lane 5 executes
    sel = lane5 & (np.arange(len(recs)) % 7 == 0)
    words[sel, 4 + 5] += np.uint64(1 << 20)                    # 1 MB away: these need the long form
    long_mask = np.random.default_rng(1).random(len(recs)) < 0.3
    slots = _encode_compact128(recs, long_mask)
    dec = nb.nvbt_decode_compact(slots, record_bytes=128)
    assert dec.shape == recs.shape and (dec == recs).all()
    with pytest.raises(nb.NvbtError):          # a long record without its continuation slots is rejected
        nb.nvbt_decode_compact(slots[(slots[:, 27] & 0xE0) == 0x40][:1], record_bytes=128)
    # skip slots between records (never inside a long record) decode to nothing
    with_skips = _with_skip_slots(slots, 128, seed=7)
    assert len(with_skips) > len(slots)
    assert np.array_equal(nb.nvbt_decode_compact(with_skips, record_bytes=128), dec)


def test_channel_bytes_layout():
    """nvbt_channel_bytes follows include/nvbt.h: 64-byte header, then per slot the record (compact: 176 B
    padded to 192) plus a 4-byte commit tag for pinned host rings; device rings (F2) carry no tag array."""
    lib = C.CDLL(LIB)
    f = lib.nvbt_channel_bytes
    f.argtypes, f.restype = [C.c_uint32, C.c_uint64, C.c_int], C.c_size_t
    assert f(288, 5, 0) == 64 + 5 * 292
    assert f(176, 7, 0) == 64 + 7 * (192 + 4)      # compact slots padded to a 192 B stride
    assert f(288, 1 << 22, 1) == 64 + 288 * (1 << 22)
    assert f(288, 0, 0) == 64
    assert f(128, 9, 0) == 128 + 9 * (128 + 4)     # 128 B slots: 128 B header, line-aligned slots
