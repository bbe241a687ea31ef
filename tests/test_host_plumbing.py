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
