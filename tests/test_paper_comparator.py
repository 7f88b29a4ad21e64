"""The paper-design comparator (comparators/paper_design.py) computes the same
function as the oracle: checked on CPU here (fp32 torch vs the fp64 oracle, same tolerances as the
CUDA path), on CUDA in tests/test_gpu_parity.py.  It is a timing baseline, never the product path."""
import numpy as np
import pytest
import torch

from comparators.paper_design import PaperDesignTT
from oracle import Oracle
from synth import workload as W
from tests.helpers import assert_companion

CASES = [
    ("c1", W.config("c1")),
    ("multi", W.small_config([37, 100, 5, 1000], [(3, 4, 4), (5, 4, 5), (1, 2, 3), (10, 10, 10)],
                             (2, 3, 2), 5, 33, 2, 1.05)),
    ("r16", W.small_config([3000, 200], [(15, 15, 14), (6, 6, 6)], (2, 2, 4), 16, 40, 3, 1.05)),
]


def run_case(cfg, device, seed=3):
    torch.backends.cuda.matmul.allow_tf32 = False
    idx, off = W.make_batch(cfg, seed=seed)
    B = cfg.batch
    cores = W.make_cores(cfg, seed=seed)
    go = W.make_grad_out(cfg, B, seed=seed)
    m = PaperDesignTT(cfg.table_rows, cfg.row_factors, cfg.col_factors, cfg.rank, device)
    m.load_cores(cores)
    out = m.forward(torch.as_tensor(idx, device=device), torch.as_tensor(off), B)
    m.backward(torch.as_tensor(go, device=device))
    orc = Oracle.from_config(cfg)
    assert_companion(out.cpu().numpy(), orc.forward(cores, idx, off, B),
                     orc.forward(cores, idx, off, B, absolute=True), 1e-5, "forward")
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    for t in range(cfg.num_tables):
        for k in range(3):
            assert_companion(m.grads[t][k].cpu().numpy().reshape(g[t][k].shape), g[t][k], ga[t][k],
                             1e-4, f"dC{k+1} t{t}")


@pytest.mark.parametrize("name,cfg", CASES, ids=[c[0] for c in CASES])
def test_paper_design_matches_oracle_cpu(name, cfg):
    run_case(cfg, "cpu")


@pytest.mark.gpu
def test_paper_design_matches_oracle_cuda():
    run_case(W.config("c2"), "cuda")
