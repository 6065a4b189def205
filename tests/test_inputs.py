"""Pins for the shared seeded input generator (vbinputs) and the workload recipes."""
import numpy as np
import torch

import vbinputs as vi


def test_splitmix64_known_value_and_vector_matches_scalar():
    # splitmix64 from state 0: first output is 0xE220A8397B1DCDAF (Vigna's reference sequence)
    assert vi.splitmix64_int(0) == 0xE220A8397B1DCDAF
    xs = [0, 1, 2, 12345, 2 ** 63, 2 ** 64 - 1]
    v = vi.splitmix64(np.array(xs, dtype=np.uint64))
    assert [int(a) for a in v] == [vi.splitmix64_int(x) for x in xs]


def test_uniform_range_exact_and_logical_indexing():
    a = vi.uniform_f32(0, 3, vi.OP_A, 37, 53)
    assert a.dtype == np.float32 and a.shape == (37, 53)
    assert a.min() >= -1.0 and a.max() < 1.0
    # every value is k * 2^-23 exactly
    k = a.astype(np.float64) * 2 ** 23
    assert np.array_equal(k, np.round(k))
    # random access agrees with the full matrix
    r = np.array([0, 5, 36]); c = np.array([52, 0, 17])
    assert np.array_equal(vi.uniform_at(0, 3, vi.OP_A, 53, r, c), a[r, c])
    # different GEMM / operand / seed -> different draws
    assert not np.array_equal(a, vi.uniform_f32(0, 4, vi.OP_A, 37, 53))
    assert not np.array_equal(a, vi.uniform_f32(0, 3, vi.OP_B, 37, 53))
    assert not np.array_equal(a, vi.uniform_f32(1, 3, vi.OP_A, 37, 53))
    # mean ~ 0, var ~ 1/3
    big = vi.uniform_f32(0, 0, vi.OP_A, 400, 500)
    assert abs(big.mean()) < 0.01 and abs(big.var() - 1 / 3) < 0.01


def test_bf16_rne_matches_torch():
    x = vi.uniform_f32(0, 9, vi.OP_B, 64, 257)
    bits = vi.f32_to_bf16_bits(x)
    t = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(bits, t)
    # explicit ties: 1 + 2^-8 (exact tie) rounds to even (1.0); 1 + 3*2^-8 rounds up
    ties = np.array([1 + 2 ** -8, 1 + 3 * 2 ** -8], np.float32)
    assert list(vi.bf16_bits_to_f64(vi.f32_to_bf16_bits(ties))) == [1.0, 1 + 2 ** -6]


def test_alpha_beta_ranges():
    al, be = vi.alpha_beta(0, range(200))
    assert al.min() >= 0.5 and al.max() < 1.5 and be.min() >= -1 and be.max() < 1
    al1, be1 = vi.alpha_beta(0, [7])
    assert al1[0] == al[7] and be1[0] == be[7]
    a2, b2 = vi.alpha_beta(0, range(3), mode="conv")
    assert list(a2) == [1, 1, 1] and list(b2) == [0, 0, 0]


def test_config_recipes():
    M, N, K = vi.config_sizes("C1")
    # SURVEY.md §8(d) lists the seed-0 draw for C1
    assert list(zip(M, N, K)) == [(112, 87, 73), (46, 50, 20), (24, 17, 35), (107, 89, 119),
                                  (72, 84, 125), (98, 87, 77), (79, 121, 47), (108, 91, 16)]
    M, N, K = vi.config_sizes("C2")
    assert len(M) == 256 and M.min() >= 32 and max(M.max(), N.max(), K.max()) <= 512
    assert abs((2 * M * N * K).sum() / 1e9 - 11.12) < 0.01
    M, N, K = vi.config_sizes("C3")
    assert len(M) == 54 and (16, 784, 192) in list(zip(M, N, K))
    M, N, K = vi.config_sizes("C4")
    assert len(M) == 4096 and K.max() <= 4096 and M.max() <= 1024 and M.min() >= 16
    assert abs((2 * M * N * K).sum() / 1e12 - 4.463) < 0.001
    M, N, K = vi.config_sizes("C5")
    assert len(M) == 65536 and min(M.min(), N.min(), K.min()) >= 16 and max(M.max(), N.max(), K.max()) <= 1024
    # log-uniform: median near sqrt(16*1025) ~ 128
    assert 100 < np.median(M) < 160


def test_padded_ld():
    assert list(vi.padded_ld([1, 8, 9, 17], "bf16")) == [8, 8, 16, 24]
    assert list(vi.padded_ld([1, 4, 5], "f32")) == [4, 4, 8]


def test_c_generator_matches_numpy_reference():
    for dtype in ("f32", "bf16", "f16"):
        for (g, op, r, c) in ((0, 0, 17, 33), (70000, 2, 64, 129), (5, 1, 1, 1)):
            ref = vi.matrix(42, g, op, r, c, dtype)[1]
            fast = vi.matrix_f64_fast(42, g, op, r, c, dtype)
            assert np.array_equal(ref, fast), (dtype, g, op)
