"""The shared input generator (inputs/): reference splitmix64 vectors and exactness."""
import numpy as np

import inputs


def test_splitmix64_reference_stream():
    # splitmix64 (Steele, Lea, Flood 2014; Vigna's reference C) started from state 0.
    want = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F, 0xF88BB8A8724C81EC]
    got = [int(v) for v in inputs.splitmix64(0, np.arange(4, dtype=np.uint64))]
    assert got == want


def test_distributions_ranges_and_offsets():
    n = 1 << 16
    f = inputs.generate("f32u", n, 7)
    assert f.dtype == np.float32 and f.min() >= 0.0 and f.max() < 1.0
    s = inputs.generate("f32s", n, 7)
    assert s.min() >= -1.0 and s.max() < 1.0 and (s < 0).any()
    # exactness: every f32u value is k * 2^-24 for an integer k
    k = f.astype(np.float64) * 2.0**24
    assert np.array_equal(k, np.round(k))
    sm = inputs.generate("small", n, 7)
    assert sm.min() >= -1000 and sm.max() <= 1000
    # offset = a window of the same stream (sharding does not change values)
    full = inputs.generate("i32", 5000, 99)
    assert np.array_equal(inputs.generate("i32", 1000, 99, offset=3000), full[3000:4000])
    # chunked generation equals one-shot
    assert np.array_equal(inputs.generate("u32", 5000, 4, chunk=333), inputs.generate("u32", 5000, 4))
    it = inputs.generate("iota", 10, 0, row_len=4)
    assert it.tolist() == [1, 2, 3, 4, 1, 2, 3, 4, 1, 2]
