"""The seeded generators: determinism, chunk independence, shapes and the SDGC constants."""
import numpy as np
import pytest

from workload import rng, sdgc


def test_rng_counter_based_and_chunk_independent():
    a = rng.uniform(7, "dropout", np.arange(1000, dtype=np.uint64))
    b = np.concatenate([rng.uniform(7, "dropout", np.arange(0, 400, dtype=np.uint64)),
                        rng.uniform(7, "dropout", np.arange(400, 1000, dtype=np.uint64))])
    assert np.array_equal(a, b)
    assert 0.45 < a.mean() < 0.55 and a.min() >= 0 and a.max() < 1
    assert not np.array_equal(a, rng.uniform(8, "dropout", np.arange(1000, dtype=np.uint64)))


def test_inputs_are_row_addressable_and_binary():
    full = sdgc.gen_inputs(1024, 300)
    part = sdgc.gen_inputs(1024, 100, row0=150)
    assert np.array_equal(full[150:250], part)
    assert set(np.unique(full)) <= {0.0, 1.0}
    assert 0.18 < full.mean() < 0.30  # ~25% density (SURVEY 8(d) calibration)


def test_radix_structure():
    net = sdgc.gen_network(4096, 3, "radix")
    assert net.strides == [1, 32, 128]
    p, idx, val, b = net.layer(1)  # stride 32
    j = 100
    assert list(idx[p[j]:p[j + 1]]) == [(j + 32 * n) % 4096 for n in range(32)]
    perm = sdgc.gen_network(1024, 2, "perm")
    p, idx, _, _ = perm.layer(0)
    # every column and every row keeps exactly 32 non-zeros
    assert np.all(np.diff(p) == 32)
    assert np.all(np.bincount(idx, minlength=1024) == 32)


def test_strides_table():
    assert sdgc.radix_strides(1024) == [1, 32]
    assert sdgc.radix_strides(16384) == [1, 32, 512]
    assert sdgc.radix_strides(65536) == [1, 32, 1024, 2048]


def test_medium_network_shape():
    net = sdgc.gen_medium_network(256, 18)
    assert net.ymax == 1.0 and net.L == 18
    assert np.all(np.diff(net.ptr[:257]) == 26)
    assert (net.bias > 0).any() and (net.bias < 0).any()
    assert sdgc.medium_t(18) == 8 and sdgc.medium_t(12) == 6


def test_pack_rows_layout():
    """snicit_infer_packed's bitmap (include/snicit.h): bit j % 32, LSB first, of word j / 32; ragged N."""
    from paper_conf_icpp_jiangh0h23_b200 import pack_rows
    rs = np.random.RandomState(5)
    for N in (4, 36, 64, 100, 1024):
        Y = (rs.uniform(size=(7, N)) < 0.3).astype(np.float32) * np.float32(2.5)
        bits = pack_rows(Y, one=2.5)
        W = (N + 31) // 32
        assert bits.shape == (7, W) and bits.dtype == np.uint32
        for r in range(7):
            for j in range(N):
                assert ((int(bits[r, j // 32]) >> (j % 32)) & 1) == (Y[r, j] != 0)
    with pytest.raises(ValueError):
        pack_rows(np.array([[0.0, 0.5, 1.0, 1.0]], np.float32))
