"""SURVEY NEXT-3 in the GPU suite: the paper's case-study axes (Fig. 9) --
sequence length and batch size around the BASELINE configs -- plus GPT-Neo's local-attention layers
(P:L185), each point checked against the fp64 oracle on 256 rows (the first and last rows of every
128-row block edge of the first and last head, the rest random).  These shapes are beyond the
BASELINE configs, whose full layers test_gpu_full_layers.py compares on every row."""
import math

import numpy as np
import pytest

import oracle
import workloads as W
from tests.gpu_util import to_dev

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
from tools.sweep import points  # noqa: E402
from bench import oracle_mask_for  # noqa: E402


def _rows(cfg, n, seed):
    rng = np.random.Generator(np.random.PCG64(seed))
    edge = [0, 1, 63, 64, 127, 128, cfg.S // 2, cfg.S - 129, cfg.S - 128, cfg.S - 1]
    rows = [g * cfg.S + i for g in (0, cfg.BH - 1) for i in edge]
    rows += rng.integers(0, cfg.BH * cfg.S, size=n - len(rows)).tolist()
    return np.array(sorted(set(rows)), dtype=np.int64)


PTS = points(quick=True)


@pytest.mark.parametrize("axis,model,cfg", PTS, ids=[f"{a}-{m}-{c.name}" for a, m, c in PTS])
def test_sweep_point(axis, model, cfg):
    t = W.make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=cfg.S + cfg.B)
    q, k, v = (to_dev(x, cfg.dtype) for x in (t.q_s, t.k_s, t.v_s))
    if cfg.kind == "dense":
        mask = sr.dense_mask(cfg.kv_len)
    elif cfg.kind == "blocksparse":
        mask = sr.block_mask(W.config_layout(cfg))
    else:
        mask = sr.window_mask(cfg.window, cfg.n_global)
    for fused in (True, False):
        o = sr.call(mask, q, k, v, scale=cfg.scale, causal=cfg.causal, out_dtype=torch.float32, fused=fused)
        torch.cuda.synchronize()
        rows = _rows(cfg, 256, seed=cfg.S)
        ref = oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, rows, oracle_mask_for(cfg))
        got = o.reshape(-1, cfg.D)[torch.from_numpy(rows).cuda()].double().cpu().numpy()
        err = np.abs(got - ref).max()
        assert err <= 1e-2, (cfg.name, fused, err)
