"""Host placement of a traced rank (drivers.bind_rank_to_gpu_numa): sysfs cpulist parsing and the split of a
NUMA node's cores between the ranks whose GPUs hang off that node. CPU only."""
from paper_conf_micro_villasnk19_b200.drivers import parse_cpulist, rank_cpu_slice


def test_parse_cpulist():
    assert parse_cpulist("0-3,8,10-11\n") == [0, 1, 2, 3, 8, 10, 11]
    assert parse_cpulist("5") == [5]
    assert parse_cpulist("") == []


def test_eight_gpus_on_two_nodes_split_evenly_and_disjoint():
    node0, node1 = list(range(0, 56)), list(range(56, 112))
    gpus = [node0] * 4 + [node1] * 4
    slices = [rank_cpu_slice(gpus, d) for d in range(8)]
    assert all(len(s) == 14 for s in slices)
    assert all(set(s) <= set(node0) for s in slices[:4]) and all(set(s) <= set(node1) for s in slices[4:])
    flat = [c for s in slices for c in s]
    assert len(flat) == len(set(flat)) == 112


def test_uneven_and_restricted():
    gpus = [list(range(10))] * 3 + [list(range(10, 16))]
    s = [rank_cpu_slice(gpus, d) for d in range(4)]
    assert [len(x) for x in s] == [3, 3, 4, 6]
    assert s[3] == list(range(10, 16))
    # the process may only run on some of the node's cores: slices come from those
    r = rank_cpu_slice(gpus, 1, allowed={0, 1, 2, 3, 4, 5})
    assert r == [2, 3]
    # more ranks than allowed cores: a rank still gets somewhere to run
    assert rank_cpu_slice([[0, 1]] * 4, 0, allowed={0, 1}) == [0, 1]
    assert rank_cpu_slice([[0, 1]] * 4, 3, allowed={0, 1}) == [1]
