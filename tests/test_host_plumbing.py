"""Host-side plumbing of the bench (CPU only): NUMA binding of the process to the GPU's node."""
import os
import types

from paper_conf_sc_eilingkkflm23_b200 import parallel as P


def test_cpulist_parse():
    assert P._cpulist("0-3,8,10-11\n") == {0, 1, 2, 3, 8, 10, 11}
    assert P._cpulist("5") == {5}
    assert P._cpulist("") == set()


def _fake_sysfs(tmp_path, bdf, node, cpulist):
    d = tmp_path / "bus" / "pci" / "devices" / bdf
    d.mkdir(parents=True)
    (d / "numa_node").write_text(f"{node}\n")
    n = tmp_path / "devices" / "system" / "node" / f"node{node}"
    n.mkdir(parents=True)
    (n / "cpulist").write_text(cpulist)


def test_bind_numa_reads_the_gpu_node(tmp_path, monkeypatch):
    props = types.SimpleNamespace(pci_domain_id=0, pci_bus_id=0x1b, pci_device_id=0)
    monkeypatch.setattr(P.torch.cuda, "get_device_properties", lambda d: props)
    before = os.sched_getaffinity(0)
    mine = sorted(before)
    _fake_sysfs(tmp_path, "0000:1b:00.0", 1, f"{mine[0]}")
    try:
        r = P.bind_numa(0, sysfs=str(tmp_path))
        assert r == {"pci": "0000:1b:00.0", "numa_node": 1, "cores": 1}
        assert os.sched_getaffinity(0) == {mine[0]}
    finally:
        os.sched_setaffinity(0, before)


def test_bind_numa_without_node_leaves_affinity(tmp_path, monkeypatch):
    props = types.SimpleNamespace(pci_domain_id=0, pci_bus_id=0x2a, pci_device_id=0)
    monkeypatch.setattr(P.torch.cuda, "get_device_properties", lambda d: props)
    before = os.sched_getaffinity(0)
    assert P.bind_numa(0, sysfs=str(tmp_path))["numa_node"] is None
    d = tmp_path / "bus" / "pci" / "devices" / "0000:2a:00.0"
    d.mkdir(parents=True)
    (d / "numa_node").write_text("-1\n")
    assert P.bind_numa(0, sysfs=str(tmp_path))["numa_node"] == -1
    assert os.sched_getaffinity(0) == before


def test_bench_defaults_meet_the_timing_contract(monkeypatch):
    """bench.py with no flags: N=1, >= 3 warm-up steps, the C5 mixed workload, inputs beyond L2."""
    import sys
    import bench
    monkeypatch.setattr(sys, "argv", ["bench.py"])
    a = bench.parse_args()
    assert a.gpus == 1 and a.warmup >= 3 and a.steps >= 10 and a.impl == "crk" and a.direction == "mixed"
    cfg = bench.workload_config(a)
    assert cfg["direction"] == "mixed" and "50/50" in cfg["workload"] and "L2" in cfg["l2"]
    assert cfg["payload_per_gpu_bytes"] == 16 * 64 * (1 << 20)
    assert bench.H2D_FRAC == {"mixed": 0.5, "h2d": 1.0, "d2h": 0.0}


def test_c5_direction_mixes():
    """gen.c5_endpoint's call mix: h2d_frac 1 / 0 gives HtoD-only / DtoH-only streams; 0.5 keeps the
    default draws (the mixed stream is the same whatever the other mixes do)."""
    from paper_conf_sc_eilingkkflm23_b200 import gen
    MiB = 1 << 20
    only_h, _ = gen.c5_endpoint(0, n_streams=2, payload_per_stream=8 * MiB, h2d_budget=8 * MiB, h2d_frac=1.0)
    only_d, _ = gen.c5_endpoint(0, n_streams=2, payload_per_stream=8 * MiB, h2d_frac=0.0)
    mixed, _ = gen.c5_endpoint(0, n_streams=2, payload_per_stream=8 * MiB)
    mixed2, _ = gen.c5_endpoint(0, n_streams=2, payload_per_stream=8 * MiB, h2d_frac=0.5)
    assert all(r.kind == gen.PROC_H2D for s in only_h for r in s.records)
    assert all(r.kind == gen.PROC_D2H for s in only_d for r in s.records)
    kinds = {r.kind for s in mixed for r in s.records}
    assert kinds == {gen.PROC_H2D, gen.PROC_D2H}
    assert [(r.kind, r.size, r.xid) for s in mixed for r in s.records] == \
           [(r.kind, r.size, r.xid) for s in mixed2 for r in s.records]
    for streams in (only_h, only_d, mixed):
        assert all(sum(r.size for r in s.records) == 8 * MiB for s in streams)


def test_next2_profiles_match_the_paper_volumes():
    """NEXT-2 profiles (gen.cusolver_endpoint / histogram_endpoint) against PAPER.md:180's transfer volumes:
    cuSolverDn_LinearSolver 6.07 GiB over its 1000 iterations, histogram 64 MiB."""
    from paper_conf_sc_eilingkkflm23_b200 import gen
    streams, rb = gen.cusolver_endpoint(iterations=3, n_streams=2)
    sizes = [r.size for s in streams for r in s.records]
    assert sizes.count(900 * 900 * 8) == 3 and sizes.count(900 * 8) == 6
    per_iter = 900 * 900 * 8 + 2 * 900 * 8
    assert abs(per_iter * gen.CUSOLVER_ITERS / 2**30 - 6.07) < 0.03   # 6.05 GiB vs the paper's 6.07 GiB
    offs = sorted((r.region_off, r.size) for s in streams for r in s.records)
    assert all(a + n <= b for (a, n), (b, _) in zip(offs, offs[1:])) and offs[-1][0] + offs[-1][1] <= rb
    h, hrb = gen.histogram_endpoint()
    assert [(r.kind, r.size) for r in h[0].records] == [(gen.PROC_H2D, 64 << 20), (gen.PROC_D2H, 1024)]
