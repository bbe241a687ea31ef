"""CPU-side checks of the C ABI: the library builds, loads and exports every entry point include/crk.h
declares; the pure host helpers agree with the oracle's closed forms; no compute is launched."""
import re

import numpy as np
import pytest

import oracle as O
from paper_conf_sc_eilingkkflm23_b200 import build, crk, gen


@pytest.fixture(scope="module")
def L():
    build.build()
    return crk.lib()


def declared_symbols():
    src = open(f"{build.ROOT}/include/crk.h").read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = set(re.findall(r"\b(crk_[a-z0-9_]+)\s*\(", src))
    # the typed families are declared one per line
    return sorted(names)


def test_exports_every_declared_symbol(L):
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", crk.LIBPATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (crk_\w+)", out))
    declared = declared_symbols()
    assert len(declared) >= 35
    missing = [s for s in declared if s not in exported]
    assert not missing, missing
    for s in declared:
        assert hasattr(L, s)


def test_config_defaults(L):
    c = crk.config()
    assert c.frag_payload == 65536 and c.strict == 1 and c.max_record_bytes == 1 << 32
    assert c.tile_bytes == 32768 and c.max_jobs == 1 << 20 and c.scan_threads == 256


def test_wire_size_closed_form_matches_oracle(L):
    for n in (0, 1, 3, 4, 5, 65503, 65504, 65505, 1 << 20, (1 << 30)):
        for F in (4, 100, 3996, 65536):
            for err in (0, 1):
                got = crk.wire_size_d2h(n, err, F)
                want = len(O.encode_memcpy_d2h(1, bytes(n) if err == 0 and n < (1 << 21) else None, err, F)) \
                    if (err or n < (1 << 21)) else O.wire_size(32 + n + (-n) % 4, F)
                assert got == want, (n, F, err)


def test_call_logical_size_matches_oracle(L):
    import torch
    ctx_items = [(crk.K_U64, 5), (crk.K_OPAQUE_VAR, torch.zeros(13, dtype=torch.uint8)), (crk.K_U32, 7),
                 (crk.K_F64_VAR, torch.zeros(3, dtype=torch.float64)),
                 (crk.K_I32_FIX | (4 << 8), torch.zeros(4, dtype=torch.int32))]
    arr, _ = crk.Context._items(ctx_items)
    n = L.crk_call_logical_size(arr, len(ctx_items))
    cfg = O.Config()
    want = len(O.call_header(1, 1, 1, 1) + O.put_u64(5) + O.put_opaque_var(bytes(13)) + O.put_u32(7)
               + O.put_array(np.zeros(3, np.float64)) + O.put_array(np.zeros(4, np.int32), False))
    assert n == want


def test_strerror_and_status_numbers_match_oracle(L):
    for name in ("OK", "INCOMPLETE", "E_ARG", "E_TRUNCATED", "E_FRAG", "E_RPC", "E_AUTH", "E_PAD", "E_SIZE",
                 "E_TRAILING", "E_XID", "E_PTR", "E_CAPACITY", "E_PROC"):
        assert getattr(crk, name) == getattr(O, name)
        assert crk.strerror(getattr(crk, name)) != "unknown status"
    for k in range(1, 17):
        assert crk.ELEM_SIZE.get(k, 0) == O.ELEM_SIZE.get(k, 0)


def test_ctx_create_without_gpu_fails_cleanly(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(crk.CrkError) as e:
        crk.Context(0)
    assert e.value.status in (crk.E_CUDA, crk.E_ARG)


def test_generator_is_deterministic():
    a, _ = gen.c5_endpoint(3, n_streams=2, payload_per_stream=1 << 22)
    b, _ = gen.c5_endpoint(3, n_streams=2, payload_per_stream=1 << 22)
    assert [(r.kind, r.xid, r.size, r.region_off) for s in a for r in s.records] == \
           [(r.kind, r.xid, r.size, r.region_off) for s in b for r in s.records]
    assert gen.c3_payload(12).tobytes() == gen.c3_payload(12).tobytes()


def test_ctypes_layouts_match_the_header(tmp_path):
    """The binding's ctypes mirrors of the public structs have the header's sizes and field offsets (gcc
    compiles a probe against include/crk.h; no CUDA headers needed)."""
    import ctypes as C
    import subprocess
    structs = {"crk_config": crk.Config, "crk_ring": crk.CRing, "crk_ring_result": crk.RingResult,
               "crk_index_view": crk.IndexView, "crk_item_req": crk.ItemReq, "crk_item_src": crk.ItemSrc,
               "crk_reply_req": crk.ReplyReq, "crk_server_bell": crk.ServerBell}
    lines = ["#include <stdio.h>", "#include <stddef.h>", '#include "crk.h"', "int main(void) {"]
    for cname, py in structs.items():
        lines.append(f'  printf("{cname} size %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'  printf("{cname} {f} %zu\\n", offsetof({cname}, {f}));')
    lines += ["  return 0;", "}"]
    src = tmp_path / "probe.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "probe"
    subprocess.run(["gcc", "-std=c11", f"-I{build.ROOT}/include", "-o", str(exe), str(src)], check=True)
    got = {}
    for line in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.splitlines():
        name, field, val = line.split()
        got[(name, field)] = int(val)
    for cname, py in structs.items():
        assert got[(cname, "size")] == C.sizeof(py), cname
        for f, _ in py._fields_:
            assert got[(cname, f)] == getattr(py, f).offset, (cname, f)


def test_config_rejects_unknown_fields(L):
    with pytest.raises(KeyError):
        crk.config(mover_reserve=16)  # misspelt: the field is mover_reserve_ctas
    assert crk.config(mover_reserve_ctas=16).mover_reserve_ctas == 16


def test_one_cta_kernels_keep_a_small_stack(L):
    """The small-step kernels (persistent server, fused front end) run one CTA whose latency is the product: taking a
    kernel parameter's address (or passing a big struct to an out-of-line helper) copies it to local memory in every
    thread at entry, which cost the front end ~80 us per launch once.  Their frames stay under 1 KiB; no kernel
    spills registers to local memory."""
    import shutil
    import subprocess
    tool = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    out = subprocess.run([tool, "-res-usage", crk.LIBPATH], capture_output=True, text=True).stdout
    usage = re.findall(r"Function (\S+):\s*\n\s*REG:(\d+) STACK:(\d+) SHARED:\d+ LOCAL:(\d+)", out)
    assert len(usage) >= 10, out[:400]
    small = {n: int(st) for n, _, st, _ in usage if "server_kernel" in n or "front_small_kernel" in n}
    assert len(small) >= 2 and all(v < 1024 for v in small.values()), small
    assert all(int(loc) == 0 for _, _, _, loc in usage), [u for u in usage if int(u[3])]
