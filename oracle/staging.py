"""Oracle staging format + pack / unpack (test infrastructure only).

PAPER.md:744-761 (section 3.3): the preempted job's state is copied to the new
device "using asynchronous memory copy"; the paper does not fix a wire format.
Format (reading Q17 in DESIGN.md), all little-endian:

    header  (32 B): magic 'SFST' | u32 version = 1 | u32 n | u32 k | u64 iter | u64 total
    entries (24 B each, n of them, ascending tensor id):
                    u32 tensor_id | u32 dtype | u64 offset | u64 nbytes
    payloads: payload i at ``offset_i``; offset_0 = round_up(32 + 24 n, 256),
              offset_{i+1} = offset_i + round_up(nbytes_i, 256);
              total = offset_{n-1} + round_up(nbytes_{n-1}, 256)  (or offset_0 if n = 0).
    Every byte not covered by the header, an entry or a payload is 0x00.

The header holds no pointers, so the bytes are device-independent: any conforming
packer produces identical bytes for the same tensor contents.

Pins (tests/test_oracle_staging.py): offsets/alignment/zero padding checked by
parsing with ``struct`` independently of this module's writer; round trip; the
empty live set; byte-exact golden fixture for a tiny hand-computed case.
"""
from __future__ import annotations

import struct
from typing import Dict, List, Tuple

import numpy as np

MAGIC = b"SFST"
VERSION = 1
ALIGN = 256
HDR_FMT = "<4sIIIQQ"
ENT_FMT = "<IIQQ"
HDR_BYTES = struct.calcsize(HDR_FMT)   # 32
ENT_BYTES = struct.calcsize(ENT_FMT)   # 24


def round_up(x: int, a: int = ALIGN) -> int:
    return (x + a - 1) // a * a


def layout(nbytes_list: List[int]) -> Tuple[List[int], int]:
    """Payload offsets and total staging size for payload sizes in entry order."""
    off = round_up(HDR_BYTES + ENT_BYTES * len(nbytes_list))
    offs = []
    for nb in nbytes_list:
        offs.append(off)
        off += round_up(nb)
    return offs, off


def pack(g, ids: List[int], T: Dict[int, np.ndarray], k: int, it: int) -> bytes:
    """Gather the live tensors ``ids`` (ascending) into one staging buffer."""
    ids = list(ids)
    assert ids == sorted(ids)
    nbs = [g.tensors[i].nbytes for i in ids]
    offs, total = layout(nbs)
    buf = bytearray(total)
    struct.pack_into(HDR_FMT, buf, 0, MAGIC, VERSION, len(ids), k, it, total)
    for e, (i, o, nb) in enumerate(zip(ids, offs, nbs)):
        struct.pack_into(ENT_FMT, buf, HDR_BYTES + ENT_BYTES * e, i, g.tensors[i].dtype, o, nb)
        raw = np.ascontiguousarray(T[i]).tobytes()
        assert len(raw) == nb, (g.tensors[i].name, len(raw), nb)
        buf[o:o + nb] = raw
    return bytes(buf)


def parse(buf: bytes):
    """Header tuple and entry list of a staging buffer."""
    magic, ver, n, k, it, total = struct.unpack_from(HDR_FMT, buf, 0)
    if magic != MAGIC or ver != VERSION:
        raise ValueError("not a staging buffer")
    ents = [struct.unpack_from(ENT_FMT, buf, HDR_BYTES + ENT_BYTES * e) for e in range(n)]
    return (magic, ver, n, k, it, total), ents


def unpack(g, buf: bytes, T: Dict[int, np.ndarray]) -> Tuple[int, int]:
    """Scatter every entry of ``buf`` into ``T`` (the target device's tensors)."""
    (_, _, n, k, it, total), ents = parse(buf)
    for (tid, dt, off, nb) in ents:
        t = g.tensors[tid]
        assert t.dtype == dt and t.nbytes == nb
        dtype = np.float32 if dt == 0 else np.int32
        T[tid] = np.frombuffer(buf[off:off + nb], dtype=dtype).reshape(t.rows, t.cols).copy()
    return k, it
