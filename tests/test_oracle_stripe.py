"""Pins the oracle's striped-memcpy rule (reading R22: Cricket's parallel-socket
memcpy) to things other than itself.  CPU only.

* The stripe CALL's wire format is built with xdrlib (an independent encoder) and parsed at xdrlib's offsets.
* decode(stripe(x)) = x: a memcpy split at random points over k rings (shuffled, interleaved with other
  calls) lands byte for byte at ptr (a numpy slice check, not the oracle's own copy routine).
* Exactly one reply per complete memcpy, on the ring of its offset-0 stripe, equal to REPLY(parent) | 0 spelled
  out with xdrlib; no stripe has a reply of its own.
* Incomplete / inconsistent memcpys (a stripe missing, a total that disagrees, a stripe outside the memcpy or the
  region) get no reply, and only their valid stripes land."""
import struct
import warnings

import numpy as np
import pytest

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import gen

with warnings.catch_warnings():
    warnings.simplefilter("ignore", DeprecationWarning)
    import xdrlib

CFG = O.Config(prog=gen.PROG, vers=gen.VERS, proc_h2d=gen.PROC_H2D, proc_d2h=gen.PROC_D2H, frag_payload=4096)
STRIPE = CFG.proc_stripe
BASE = 0x7F0000000000


def stripe_call(xid, ptr, data, offset, total, parent, size=None, F=4096):
    return O.encode_call(xid, STRIPE, [(O.K_U64, ptr), (O.K_OPAQUE_VAR, bytes(data)),
                                       (O.K_U64, len(data) if size is None else size), (O.K_U32, parent),
                                       (O.K_U64, offset), (O.K_U64, total)], CFG, F=F)


def reply_wire(xid, err=0, F=4096):
    p = xdrlib.Packer()
    for v in (xid, 1, 0, 0, 0, 0, err):
        p.pack_uint(v)
    L = p.get_buffer()
    return struct.pack(">I", 0x80000000 | len(L)) + L  # one fragment (28 < F)


def serve(ring_wires, region_bytes=1 << 16):
    rings = []
    for ws in ring_wires:
        w = b"".join(ws)
        ring = np.zeros(1 << max(8, len(w).bit_length()), np.uint8)
        ring[:len(w)] = np.frombuffer(w, np.uint8)
        rings.append((ring, 0, len(w)))
    region = np.zeros(region_bytes, np.uint8)
    out = O.serve(rings, CFG, region, BASE, [1 << 14] * len(rings), [0] * len(rings))
    assert all(s == O.OK for s in out["scan_status"])
    return out, region


def test_stripe_wire_format_vs_xdrlib():
    data = bytes(range(7))
    p = xdrlib.Packer()
    for v in (0x51, 0, 2, gen.PROG, gen.VERS, STRIPE, 0):
        p.pack_uint(v)
    p.pack_opaque(b"")
    p.pack_uint(0)
    p.pack_opaque(b"")
    p.pack_uhyper(BASE + 8)
    p.pack_opaque(data)
    p.pack_uhyper(7)
    p.pack_uint(0xAB)
    p.pack_uhyper(100)
    p.pack_uhyper(4000)
    L = p.get_buffer()
    assert O.frame(L, 4096) == stripe_call(0x51, BASE + 8, data, 100, 4000, 0xAB)
    c = O.parse_call(L, CFG)
    assert c.status == O.OK and c.proc == STRIPE and c.n_items == 6
    assert (c.value[0], c.count[1], c.off[1], c.value[2]) == (BASE + 8, 7, 52, 7)
    assert (c.value[3], c.value[4], c.value[5]) == (0xAB, 100, 4000)


@pytest.mark.parametrize("seed", range(8))
def test_striped_memcpy_lands_and_completes_once(seed):
    g = gen.rng(seed)
    total = int(g.integers(1, 30000))
    payload = gen.random_bytes(seed, total)
    k = int(g.integers(1, 9))
    cuts = sorted(set(int(x) for x in g.integers(0, total, k - 1))) if k > 1 else []
    bounds = [0] + cuts + [total]
    stripes = [(a, b) for a, b in zip(bounds, bounds[1:])]
    n_rings = int(g.integers(1, 5))
    ptr = BASE + 1000 + int(g.integers(0, 16))
    parent = 0xC0DE0000 + seed
    ring_wires = [[] for _ in range(n_rings)]
    lead_ring, others = None, 0
    for s, i in enumerate(g.permutation(len(stripes)).tolist()):
        a, b = stripes[i]
        r = int(g.integers(0, n_rings))
        if g.random() < 0.4:  # an unrelated DtoH call in between
            ring_wires[r].append(O.encode_call(0xD0000 + others, gen.PROC_D2H, [(O.K_U64, BASE), (O.K_U64, 8)], CFG,
                                               F=4096))
            others += 1
        ring_wires[r].append(stripe_call(0x5000 + s, ptr, payload[a:b], a, total, parent))
        if a == 0:
            lead_ring = r
    out, region = serve(ring_wires)
    o = ptr - BASE
    assert region[o:o + total].tobytes() == payload.tobytes()  # decode(stripe(x)) == x
    assert not region[:o].any() and not region[o + total:].any()
    stripes_out = [r for r in out["records"] if r["proc"] == STRIPE]
    assert all(r["status"] == O.OK for r in stripes_out)
    with_reply = [r for r in stripes_out if r["reply_err"] >= 0]
    assert len(with_reply) == 1 and with_reply[0]["ring"] == lead_ring  # one reply, from the offset-0 stripe
    rr = with_reply[0]
    send = out["send"][lead_ring]
    assert bytes(send[rr["reply_off"]:rr["reply_off"] + rr["reply_wire"]]) == reply_wire(parent)


def test_incomplete_or_inconsistent_memcpys_get_no_reply():
    payload = gen.random_bytes(77, 5000)
    parts = [(0, 2000), (2000, 3500), (3500, 5000)]

    def calls(parent, skip=None, total=5000, bad_total_at=None, ptr=BASE + 64):
        ws = []
        for i, (a, b) in enumerate(parts):
            if i == skip:
                continue
            t = total + 1 if i == bad_total_at else total
            ws.append(stripe_call(parent * 16 + i, ptr, payload[a:b], a, t, parent))
        return ws
    # a stripe missing: no reply; the others land
    out, region = serve([calls(1, skip=1)])
    assert all(r["reply_err"] == -1 for r in out["records"])
    assert region[64:64 + 2000].tobytes() == payload[:2000].tobytes() and not region[64 + 2000:64 + 3500].any()
    assert region[64 + 3500:64 + 5000].tobytes() == payload[3500:].tobytes()
    # the lead missing: the bytes all land except its own, no reply
    out, _ = serve([calls(2, skip=0)])
    assert all(r["reply_err"] == -1 for r in out["records"])
    # one stripe claims another total: inconsistent, no reply
    out, _ = serve([calls(3, bad_total_at=2)])
    assert all(r["reply_err"] == -1 for r in out["records"])
    # stripe checks: past the memcpy's total -> E_SIZE, outside the region -> E_PTR, size != n -> E_SIZE
    bad = [stripe_call(0x901, BASE, payload[:10], 4995, 5000, 9),
           stripe_call(0x902, BASE + (1 << 16) - 4, payload[:10], 0, 10, 10),
           stripe_call(0x903, BASE, payload[:10], 0, 10, 11, size=11)]
    out, region = serve([bad])
    assert [r["status"] for r in out["records"]] == [O.E_SIZE, O.E_PTR, O.E_SIZE]
    assert all(r["reply_err"] == -1 for r in out["records"]) and not region.any()


def test_two_memcpys_interleaved_over_rings_and_disabled_proc():
    a, b = gen.random_bytes(5, 3000), gen.random_bytes(6, 7000)
    r0 = [stripe_call(1, BASE, a[:1000], 0, 3000, 0xA), stripe_call(2, BASE + 4096, b[4000:], 4000, 7000, 0xB)]
    r1 = [stripe_call(3, BASE + 4096, b[:4000], 0, 7000, 0xB), stripe_call(4, BASE, a[1000:], 1000, 3000, 0xA)]
    out, region = serve([r0, r1])
    assert region[:3000].tobytes() == a.tobytes() and region[4096:4096 + 7000].tobytes() == b.tobytes()
    rep = [(r["ring"], r["xid"]) for r in out["records"] if r["reply_err"] == 0]
    assert rep == [(0, 1), (1, 3)]  # each memcpy's offset-0 stripe carries its reply
    assert bytes(out["send"][0][:32]) == reply_wire(0xA) and bytes(out["send"][1][:32]) == reply_wire(0xB)
    # with the stripe procedure disabled the same CALLs are an unknown procedure (reading R20)
    cfg_off = O.Config(**{**CFG.__dict__, "proc_stripe": 0})
    w = b"".join(r0)
    ring = np.zeros(1 << 15, np.uint8)
    ring[:len(w)] = np.frombuffer(w, np.uint8)
    out = O.serve([(ring, 0, len(w))], cfg_off, np.zeros(1 << 16, np.uint8), BASE, [1 << 14], [0])
    assert [r["status"] for r in out["records"]] == [O.E_PROC, O.E_PROC]
