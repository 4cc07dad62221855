"""Host-side check of the counted reduction tree's index arithmetic (the carry
mechanism of the integer pairs, csrc/sat_kernel.cuh tree_update / tree_query /
tree_release), written out independently in Python: for
every (bands per image, images, cluster size) the per-image Fenwick nodes that
clusters contribute to and read must give each cluster exactly the sum of the
band contributions above it in its image (the carry into a
block is the column total of everything above it), every node must receive
exactly lowbit(i) contributions (the completeness count a reader checks), be
read by exactly min(lowbit(i), D - i) clusters (the last of them zeroes it),
and node storage of different images must not overlap."""
import random

import pytest


def lowbit(i):
    return i & -i


def simulate(bpi, batch, CL, seed=0):
    rng = random.Random(seed)
    nb = bpi * batch
    tickets = (nb + CL - 1) // CL
    first = lambda n: (n * bpi) // CL                          # img_first_ticket
    count = lambda n: ((n + 1) * bpi - 1) // CL - (n * bpi) // CL + 1  # img_tickets
    val = [rng.randrange(1 << 20) for _ in range(nb)]  # band column totals (one column)
    node, writes, reads = {}, {}, {}
    for T in range(tickets):  # tree_update: the tail segment's contribution
        g0, glast = T * CL, min(T * CL + CL, nb) - 1
        nt = glast // bpi
        contrib = sum(val[g] for g in range(g0, glast + 1) if g // bpi == nt)
        t, D = T - first(nt), count(nt)
        has_succ = glast % bpi + 1 < bpi
        assert has_succ == (t < D - 1)
        i = t + 1
        while i <= D - 1:
            key = first(nt) + i - 1
            node[key] = node.get(key, 0) + contrib
            writes[key] = writes.get(key, 0) + 1
            i += lowbit(i)
    for T in range(tickets):  # tree_query of the head image
        g0 = T * CL
        n0, k0 = g0 // bpi, g0 % bpi
        if k0 == 0:
            continue  # the cluster starts its image: carry = the image's carry-in row
        t = T - first(n0)
        assert t >= 1
        total, i = 0, t
        while i > 0:
            key = first(n0) + i - 1
            assert writes.get(key, 0) == lowbit(i)  # the node is complete when read
            total += node[key]
            reads[key] = reads.get(key, 0) + 1
            i -= lowbit(i)
        assert total == sum(val[g] for g in range(n0 * bpi, g0))
    for n in range(batch):  # tree_release: reader counts; storage ranges per image
        D = count(n)
        for i in range(1, D):
            key = first(n) + i - 1
            assert reads.get(key, 0) == min(lowbit(i), D - i)
            assert key < first(n) + D - 1 <= (first(n + 1) if n + 1 < batch else tickets)
    return tickets


@pytest.mark.parametrize("CL", [1, 2, 4, 5, 8])
@pytest.mark.parametrize("batch", [1, 2, 3, 7])
@pytest.mark.parametrize("bpi", [1, 2, 3, 4, 5, 6, 7, 9, 16, 33, 34, 100, 512, 513])
def test_tree_indices(bpi, batch, CL):
    simulate(bpi, batch, CL, seed=bpi * 131 + batch * 7 + CL)


def test_tree_depth_of_the_benchmark_shapes():
    # 16384^2 8u (512 bands, clusters of 5): 103 clusters, <= 7 nodes per query
    assert simulate(512, 1, 5) == 103
    assert max(bin(t).count("1") for t in range(1, 103)) == 6
    # 1080p batch (34 bands per frame, clusters of 5, frames straddling clusters)
    simulate(34, 64, 5)
