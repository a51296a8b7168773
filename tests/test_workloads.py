"""The torch generator equals the numpy generator bit for bit (they feed the GPU and the oracle)."""
import numpy as np
import torch

import workloads as W


def test_splitmix_torch_equals_numpy():
    idx = np.arange(0, 1 << 16, dtype=np.uint64) * np.uint64(7919)
    a = W.splitmix64(W.key(5, 3), idx)
    b = W.splitmix64_t(W.key(5, 3), torch.from_numpy(idx.view(np.int64))).numpy().view(np.uint64)
    assert (a == b).all()


def test_queries_torch_equals_numpy():
    offs, sizes, span = W.table_layout(1 << 14, 5)
    q, u = W.queries(offs, sizes, 100003, 5, start=12345)
    qt, ut = W.queries_t(torch.from_numpy(offs.view(np.int64)), torch.from_numpy(sizes.view(np.int64)),
                         100003, 5, start=12345, chunk=40000)
    assert (qt.numpy().view(np.uint64) == q).all() and (ut.numpy() == u.astype(np.int64)).all()


def test_table_layout_shape():
    offs, sizes, span = W.table_layout(1 << 16, 3)
    assert sizes.min() >= 16 and sizes.max() < 65536 and (sizes % 16 == 0).all()
    gaps = offs[1:] - (offs[:-1] + sizes[:-1])
    assert gaps.max() <= 4080 and (gaps % 16 == 0).all()
    assert 0.002 < (gaps == 0).mean() < 0.007          # adjacency with p = 1/256
    assert 7000 < sizes.mean() < 8800                    # log-uniform mean 16*4095/ln 4096 = 7877
