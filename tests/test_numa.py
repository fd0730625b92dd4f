"""NUMA host logic of the pinned store ("Placement SPLIT (layer k -> node k mod n;
Adam threads of that node) or LOCAL (GPU's node); DP: slice r of every layer on GPU r's node").

The build box has one NUMA node, so the multi-node plan is exercised against fake sysfs trees
(SH_SYSFS_ROOT) and the placement primitive (mbind before first touch, read back with
get_mempolicy) on the real node 0.  CPU only."""
import os

import pytest

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")


def _fake_sysfs(tmp_path, nodes: dict[int, str], pci: dict[str, str] | None = None):
    k = 0
    while (tmp_path / f"sysfs{k}").exists():
        k += 1
    root = tmp_path / f"sysfs{k}"
    base = root / "sys/devices/system/node"
    base.mkdir(parents=True)
    ids = sorted(nodes)
    (base / "online").write_text(",".join(str(i) for i in ids) + "\n")
    for i, cl in nodes.items():
        (base / f"node{i}").mkdir()
        (base / f"node{i}" / "cpulist").write_text(cl + "\n")
    for bus, node in (pci or {}).items():
        d = root / "sys/bus/pci/devices" / bus
        d.mkdir(parents=True)
        (d / "numa_node").write_text(node + "\n")
    return str(root)


@pytest.fixture
def sysfs(tmp_path, monkeypatch):
    def make(nodes, pci=None):
        monkeypatch.setenv("SH_SYSFS_ROOT", _fake_sysfs(tmp_path, nodes, pci))
    yield make
    monkeypatch.delenv("SH_SYSFS_ROOT", raising=False)
    sh.numa_topology()  # re-read the real topology for later tests


def test_topology_parses_cpulists(sysfs):
    sysfs({0: "0-23,48-71", 1: "24-47,72-95"})  # the paper's 2 x 24-core Xeon with SMT
    assert sh.numa_topology() == [(0, 48), (1, 48)]
    sysfs({0: "0,2,4-5", 3: "1,3"})  # sparse node ids, singletons
    assert sh.numa_topology() == [(0, 4), (3, 2)]


def test_topology_without_sysfs_is_one_node(tmp_path, monkeypatch):
    monkeypatch.setenv("SH_SYSFS_ROOT", str(tmp_path / "nothing"))
    topo = sh.numa_topology()
    assert len(topo) == 1 and topo[0][1] == os.cpu_count()
    monkeypatch.delenv("SH_SYSFS_ROOT")


def test_real_topology_counts_every_cpu():
    topo = sh.numa_topology()
    assert len(topo) >= 1 and sum(c for _, c in topo) == os.cpu_count()


def test_plan_split_local_interleave():
    n = 2
    # SPLIT: layer k -> node k mod n
    assert [sh.numa_plan(sh.SH_NUMA_SPLIT, k, n) for k in range(6)] == [0, 1, 0, 1, 0, 1]
    assert [sh.numa_plan(sh.SH_NUMA_SPLIT, k, 3) for k in range(6)] == [0, 1, 2, 0, 1, 2]
    # LOCAL: every layer on the GPU's node
    assert {sh.numa_plan(sh.SH_NUMA_LOCAL, k, n, gpu_node=1) for k in range(6)} == {1}
    # INTERLEAVE: -2, NONE: -1
    assert sh.numa_plan(sh.SH_NUMA_INTERLEAVE, 3, n) == -2
    assert sh.numa_plan(sh.SH_NUMA_NONE, 3, n) == -1
    # one node: never bound, whatever the policy
    for pol in range(5):
        assert sh.numa_plan(pol, 5, 1) == -1


def test_plan_auto_resolution():
    # private store on a multi-node host: SPLIT; shared (data-parallel) store: LOCAL (slice r on
    # GPU r's node); single node: nothing
    assert [sh.numa_plan(sh.SH_NUMA_AUTO, k, 2) for k in range(4)] == [0, 1, 0, 1]
    assert [sh.numa_plan(sh.SH_NUMA_AUTO, k, 2, gpu_node=1, shared=True) for k in range(4)] == [1, 1, 1, 1]
    assert sh.numa_plan(sh.SH_NUMA_AUTO, 0, 1) == -1


def test_worker_nodes_follow_core_counts(sysfs):
    sysfs({0: "0-3", 1: "4-7"})
    nodes = [sh.numa_worker_node(sh.SH_NUMA_SPLIT, t, 8) for t in range(8)]
    assert nodes == [0, 1, 0, 1, 0, 1, 0, 1]
    # unequal nodes: workers in proportion to cores (6 : 2)
    sysfs({0: "0-5", 1: "6-7"})
    nodes = [sh.numa_worker_node(sh.SH_NUMA_SPLIT, t, 8) for t in range(8)]
    assert nodes.count(0) == 6 and nodes.count(1) == 2
    # LOCAL: all on the GPU's node; INTERLEAVE / NONE: unpinned
    assert {sh.numa_worker_node(sh.SH_NUMA_LOCAL, t, 8, gpu_node=1) for t in range(8)} == {1}
    assert {sh.numa_worker_node(sh.SH_NUMA_INTERLEAVE, t, 8) for t in range(8)} == {-1}
    # AUTO on a multi-node host with a private store = SPLIT
    assert [sh.numa_worker_node(sh.SH_NUMA_AUTO, t, 4) for t in range(4)] == [0, 1, 0, 1]


def test_worker_nodes_single_node_unpinned(sysfs):
    sysfs({0: "0-15"})
    assert {sh.numa_worker_node(p, t, 16) for p in range(5) for t in range(16)} == {-1}


def test_gpu_node_from_pci_sysfs(sysfs):
    sysfs({0: "0-7", 1: "8-15"}, pci={"0000:1b:00.0": "1", "0000:9a:00.0": "0", "0000:aa:00.0": "-1"})
    assert sh.numa_node_of_pci("0000:1B:00.0") == 1  # cudaDeviceGetPCIBusId prints upper case
    assert sh.numa_node_of_pci("0000:9a:00.0") == 0
    assert sh.numa_node_of_pci("0000:aa:00.0") == 0  # no affinity -> node index 0
    assert sh.numa_node_of_pci("0000:ff:00.0") == 0  # unknown device
    # sparse node ids map to indices
    sysfs({0: "0-7", 2: "8-15"}, pci={"0000:1b:00.0": "2"})
    assert sh.numa_node_of_pci("0000:1b:00.0") == 1


def test_mbind_places_pages_on_the_requested_node():
    """The placement primitive the store uses: mbind before the first touch, read back per page."""
    node = sh.numa_topology()[0][0]
    got = sh.numa_bind_check(node, 8 << 20)
    if got == -1:
        pytest.skip("mbind/get_mempolicy not permitted in this container")
    assert got == node
