"""Input generator checks (CPU): Philox4x32-10 known answers, determinism and
the structural properties of the synthetic workloads (DESIGN.md input recipe)."""
import numpy as np

import graphgen


def test_philox_known_answers():
    # Random123 kat_vectors, philox4x32 with 10 rounds.
    assert graphgen.philox_block([0, 0, 0, 0], [0, 0]).tolist() == [
        0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]
    assert graphgen.philox_block([0xFFFFFFFF] * 4, [0xFFFFFFFF] * 2).tolist() == [
        0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD]
    assert graphgen.philox_block([0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344],
                                 [0xA4093822, 0x299F31D0]).tolist() == [
        0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]


def test_deterministic_across_threads_and_offsets():
    spec = graphgen.rmat_spec(14, 8, 99)
    a = graphgen.generate_cpu(spec, threads=1)
    b = graphgen.generate_cpu(spec, threads=7)
    assert all(np.array_equal(x, y) for x, y in zip(a, b))
    c = graphgen.generate_cpu(spec, e0=1000, count=500)
    assert np.array_equal(c[0], a[0][1000:1500]) and np.array_equal(c[1], a[1][1000:1500])


def test_rmat_range_and_skew():
    spec = graphgen.rmat_spec(14, 16, 5)
    s, d = graphgen.generate_cpu(spec)
    assert s.max() < spec.n and d.max() < spec.n
    deg = np.bincount(np.concatenate([s, d]), minlength=spec.n)
    assert deg.max() > 50 * deg.mean()  # power-law skew


def test_scramble_is_bijection():
    spec = graphgen.rmat_spec(10, 1, 3, scramble=True)
    raw = graphgen.rmat_spec(10, 1, 3, scramble=False)
    s1, _ = graphgen.generate_cpu(spec)
    s0, _ = graphgen.generate_cpu(raw)
    # same pre-image -> same image, different pre-image -> different image
    mp = {}
    for a, b in zip(s0.tolist(), s1.tolist()):
        assert mp.setdefault(a, b) == b
    assert len(set(mp.values())) == len(mp)


def test_er_range_uniform():
    spec = graphgen.er_spec(1000, 200000, 8)
    s, d = graphgen.generate_cpu(spec)
    assert s.max() < 1000 and d.max() < 1000
    deg = np.bincount(np.concatenate([s, d]), minlength=1000)
    assert deg.max() < 2 * deg.mean()
