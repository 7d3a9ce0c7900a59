"""N4: host-resident feature tables + preload().

The operand tables live in pinned host memory; every block copies the rows it gathers
(edge rows by eid, the tail block's node rows by nbr / dst) into device staging tables
with tgl_preload_rows -- the GPU reads host memory directly -- and runs the same kernels
on them with identity indices.  The embeddings must equal the all-on-GPU pipeline's BIT
FOR BIT (same values, same kernels, same reduction order), eager and graph-replayed, in
both operand layouts, with dedup on and off.
"""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("name,layout", [("REDDIT", "split"), ("REDDIT", "fp32"),
                                         ("WIKI", "split"), ("GDELT", "split")])
def test_host_features_equal_device(name, layout):
    from paper_conf_asplos_wangm24_b200 import TGATPipeline, TSampler, tgl
    cfg = synth.get_config(name).scaled(60000, batch=300)
    g = synth.make_graph(cfg)
    neg = synth.make_negatives(cfg)
    params = synth.gen.model_params(cfg)

    def pitch4(a):                       # 16-byte row pitch (the fp32 K|V path needs it)
        n, d = a.shape
        t = torch.zeros(n, (d + 3) // 4 * 4, dtype=torch.float32, device="cuda")
        t[:, :d] = cu(a)
        return t[:, :d]
    dev = {"src": cu(g.src), "dst": cu(g.dst), "t": cu(g.t), "neg": cu(neg),
           "nfeat": pitch4(g.nfeat), "efeat": pitch4(g.efeat)}
    tc = tgl.build_tcsr(cfg.n_nodes, dev["src"], dev["dst"], dev["t"], True, True)
    mk = lambda host: TGATPipeline(dev, tc, params, cfg.batch,
                                   TSampler(cfg.k, cfg.strategy, cfg.seeds["sampler"]), cfg.dedup,
                                   cfg.precompute, cfg.window, "fp32", layout=layout,
                                   host_features=host)
    pd, ph = mk(False), mk(True)
    assert ph.nfeat_host is not None and not ph.nfeat_host.is_cuda and ph.nfeat_host.is_pinned()
    n0 = 3 * cfg.batch
    for b in (0, cfg.n_batches // 2, cfg.n_batches - 1):
        pd.start_dev.fill_(b * cfg.batch)
        ph.start_dev.fill_(b * cfg.batch)
        ed = pd.forward()[:n0].cpu().numpy().copy()
        eh = ph.forward()[:n0].cpu().numpy().copy()
        assert np.array_equal(ed, eh), (name, layout, b)
    ph.capture()
    b = int(0.7 * cfg.n_batches)
    pd.start_dev.fill_(b * cfg.batch)
    ed = pd.forward()[:n0].cpu().numpy().copy()
    eg = ph.run_graph(b * cfg.batch)[:n0].cpu().numpy()
    assert np.array_equal(ed, eg)


def test_preload_rows_from_pinned_host():
    """tgl_preload_rows: rows of a pinned host table by index, count read on the device at
    n_dev[*n_at] (a block's seg_ptr[U]); 16-byte and 4-byte row paths."""
    from paper_conf_asplos_wangm24_b200 import tgl
    rng = np.random.default_rng(1)
    for d in (104, 13):
        src = torch.from_numpy(rng.standard_normal((1000, d)).astype(np.float32)).pin_memory()
        idx = cu(rng.integers(0, 1000, 700).astype(np.int32))
        out = torch.full((700, d), -7.0, device="cuda")
        counts = cu(np.array([3, 555, 9], np.int64))
        at = cu(np.array([1], np.int64))
        tgl.preload_rows(idx, src, out, n_max=700, n_dev=counts, n_at=at)
        torch.cuda.synchronize()
        got = out.cpu().numpy()
        exp = src.numpy()[idx.cpu().numpy()[:555]]
        assert np.array_equal(got[:555], exp)
        assert (got[555:] == -7.0).all()
