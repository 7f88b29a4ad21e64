"""Host-memory tier on the GPU (PAPER §V): the pipeline with its
embedding cache computes bit-for-bit what sequential training computes (oracle/hosttier_ref.py),
for several queue lengths, with the server as a free-running thread or inline at the most stale
legal schedule; without the cache it computes the stale pipeline instead (the RAW conflict of
P:296), which differs."""
import numpy as np
import pytest
import torch

from oracle import hosttier_ref as HR
from synth import workload as W

pytestmark = pytest.mark.gpu

ROWS = [300, 50, 800]
DIM = 16
B = 32
POOL = 3
STEPS = 10
LR = 0.05
TB = np.concatenate([[0], np.cumsum(ROWS)]).astype(np.int64)


@pytest.fixture(scope="module")
def data():
    bs = [W.make_host_batch(ROWS, B, POOL, 1.05, step=k, seed=11) for k in range(STEPS)]
    ys = [0.1 * W.make_host_grad_out(len(ROWS), B, DIM, step=k, seed=11) for k in range(STEPS)]
    W0 = W.make_host_weight(ROWS, DIM, seed=11)
    seq = HR.train_sequential(W0, TB, bs, HR.squared_loss_grad(ys), B, LR)
    return bs, ys, W0, seq


def _run(data, L, threaded, use_cache, host_threads=0):
    from paper_conf_sc_wangwfmmd22_b200.hosttier import HostTierEmbedding
    bs, ys, W0, _ = data
    dev = torch.device("cuda", 0)
    ht = HostTierEmbedding(ROWS, DIM, B, len(ROWS) * B * POOL, L, LR, threaded=threaded,
                           use_cache=use_cache, server_threads=host_threads, weight=W0)
    yd = [torch.as_tensor(y, device=dev) for y in ys]
    ht.start(lambda k: bs[k], STEPS)
    outs = []
    for k in range(STEPS):
        out = ht.forward(k)
        ht.backward((out - yd[k]).contiguous())      # d(1/2|out - y|^2)/d out, float32
        outs.append(out.cpu().numpy())
    ht.finish()
    live, ovf = ht.cache_stats()
    return ht.weight.numpy().copy(), outs, live, ovf, ht


@pytest.mark.parametrize("L,threaded", [(1, True), (2, True), (4, True), (3, False), (1, False)])
def test_pipeline_with_cache_is_sequential_training(data, L, threaded):
    Wseq, oseq = data[3]
    Wp, outs, live, ovf, ht = _run(data, L, threaded, True)
    assert ovf == 0 and 0 < live <= ht.capacity
    for k in range(STEPS):
        np.testing.assert_array_equal(outs[k], oseq[k], err_msg=f"out of batch {k}")
    np.testing.assert_array_equal(Wp, Wseq)


def test_pipeline_without_cache_is_stale(data):
    bs, ys, W0, (Wseq, oseq) = data
    L = 3
    Ws, os_ = HR.train_stale(W0, TB, bs, HR.squared_loss_grad(ys), B, LR, L)
    Wp, outs, live, ovf, _ = _run(data, L, False, False)
    assert live == 0
    for k in range(STEPS):
        np.testing.assert_array_equal(outs[k], os_[k], err_msg=f"out of batch {k}")
    np.testing.assert_array_equal(Wp, Ws)
    assert not np.array_equal(Wp, Wseq)          # the RAW conflict changed the training


def test_cache_life_cycle_bound(data):
    """Live entries never exceed the rows of the last L batches; after the last batch exactly the
    rows of batches STEPS-L .. STEPS-1 are cached (each pushed with LC = L, one tick per batch)."""
    bs = data[0]
    L = 2
    _, _, live, ovf, ht = _run(data, L, False, True)
    from paper_conf_sc_wangwfmmd22_b200.hosttier import prepare_batch
    last = set()
    for k in range(STEPS - L, STEPS):
        last |= set(prepare_batch(*bs[k], TB, B).ids.tolist())
    assert ovf == 0 and live == len(last)
    idx = ht.c_index.cpu().numpy()
    assert set(np.nonzero(idx >= 0)[0].tolist()) == last
