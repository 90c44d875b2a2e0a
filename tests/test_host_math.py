"""Host-side integer arithmetic the kernels rely on (no GPU): the multiply-high
divisions by host-computed magic numbers must equal the exact quotients over
the operand ranges the dispatcher allows."""
import numpy as np


def _umulhi_div(x, d):
    m = ((1 << 32) + d - 1) // d  # ceil(2^32 / d), as tlp_agg.cu computes fh_magic
    return (x.astype(np.uint64) * np.uint64(m)) >> np.uint64(32)


def test_head_index_magic_exact_for_small_F():
    """mh_div (tlp_agg_kernels.cuh): x / fh = umulhi(x, ceil(2^32 / fh)) for
    every column x < F when F < 2^16 and 1 < fh <= F (exhaustive up to F = 1024,
    then every divisor of a few widths and all columns near multiples)."""
    for F in range(2, 1025):
        x = np.arange(F, dtype=np.uint64)
        for d in range(2, F + 1):
            assert np.array_equal(_umulhi_div(x, d), x // np.uint64(d)), (F, d)
            if d > 64:
                break  # larger divisors covered below
    rng = np.random.default_rng(0)
    for F in (1433, 4096, 30000, 65535):
        x = np.arange(F, dtype=np.uint64)
        for d in list(range(2, 200)) + list(rng.integers(200, F + 1, 200)):
            d = int(d)
            assert np.array_equal(_umulhi_div(x, d), x // np.uint64(d)), (F, d)
