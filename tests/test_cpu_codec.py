"""The multi-core CPU codec (libpfpl_cpu.so) against the oracle.

P:43: PFPL's CPU and GPU implementations produce bit-for-bit identical
compressed and decompressed output; the CPU production codec must therefore
write exactly the oracle's stream bytes and decode the oracle's streams to the
oracle's values, for every bound, dtype and size, with any thread count.
"""
import numpy as np
import pytest

import synth
from tests.boundcheck import violations


@pytest.fixture(scope="module")
def cpu():
    from paper_conf_ipps_fallinadcb25_b200 import cpu
    cpu.lib()
    return cpu


def _bits(a):
    return a.view(np.uint32 if a.dtype == np.float32 else np.uint64)


def _check(cpu, orc, x, bound, eps, ms=False, nthreads=0):
    s_cpu = cpu.compress(x, bound, eps, ms=ms, nthreads=nthreads)
    s_orc = orc.compress(x, bound, eps, ms=ms)
    assert s_cpu == s_orc, f"stream differs ({bound}, {x.dtype}, n={x.size}, eps={eps})"
    y = cpu.decompress(s_orc, nthreads=nthreads)
    assert np.array_equal(_bits(y), _bits(orc.decompress(s_orc)))
    assert violations(x, y, bound, eps).size == 0


SIZES = [1, 31, 32, 33, 2047, 2048, 2049, 4095, 4096, 4097, 3 * 4096 + 17, 20000]


@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-1, 1e-2, 1e-3, 1e-4])
def test_fields_all_sizes(cpu, orc, bound, dt, eps):
    for n in SIZES:
        spec = synth.FieldSpec("t", (n,), "f32" if dt == np.float32 else "f64", 3, A=0.5, tau=0.01)
        _check(cpu, orc, synth.generate(spec).numpy(), bound, eps)


@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-1, 1e-4, 0.37])
def test_adversarial(cpu, orc, bound, dt, eps):
    x = synth.adversarial_f32() if dt == np.float32 else synth.adversarial_f64()
    _check(cpu, orc, x, bound, eps)


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_random_bits_constants_zeros_ms(cpu, orc, dt):
    rng = np.random.default_rng(7)
    n = 5 * (16384 // np.dtype(dt).itemsize) + 3
    u = rng.integers(0, 2**63, size=n, dtype=np.int64).astype(np.uint64)
    x = (u.astype(np.uint32) if dt == np.float32 else u).view(dt)
    for bound in ("abs", "rel", "noa"):
        _check(cpu, orc, x, bound, 1e-3)
        _check(cpu, orc, np.full(n, 2.5, dt), bound, 1e-3)
        _check(cpu, orc, np.zeros(n, dt), bound, 1e-3)
        spec = synth.FieldSpec("t", (40000,), "f32" if dt == np.float32 else "f64", 5, A=1.0, tau=0.01)
        _check(cpu, orc, synth.generate(spec).numpy(), bound, 1e-3, ms=True)


@pytest.mark.parametrize("nthreads", [1, 3, 8])
def test_thread_counts_and_rough_field(cpu, orc, nthreads):
    """Dynamic chunk assignment + carry array: any thread count
    gives the same stream; the rough NYX variant exercises many active planes."""
    x = synth.generate(synth.CONFIGS["nyx_rough"], slab=(0, 2)).numpy()
    _check(cpu, orc, x, "abs", 1e-3, nthreads=nthreads)
    x = synth.generate(synth.CONFIGS["hurricane"], slab=(49, 51)).numpy()
    _check(cpu, orc, x, "rel", 1e-3, nthreads=nthreads)


def test_empty_capacity_errors(cpu, orc):
    for dt in (np.float32, np.float64):
        assert cpu.compress(np.zeros(0, dt), "abs", 1e-3) == orc.compress(np.zeros(0, dt), "abs", 1e-3)
        assert cpu.decompress(orc.compress(np.zeros(0, dt), "abs", 1e-3)).size == 0
    with pytest.raises(cpu.PFPLCPUError) as e:
        cpu.compress(np.ones(10, np.float32), "abs", 1e-40)
    assert e.value.code == -2
    for bad in (0.0, -1.0, float("nan"), float("inf")):
        with pytest.raises(cpu.PFPLCPUError):
            cpu.compress(np.ones(10, np.float32), "rel", bad)


def test_corrupt_streams_never_crash(cpu, orc):
    """Every corrupt stream decodes or returns PFPL_ERR_CORRUPT (-4); truncated and
    trailing-byte streams are rejected (P:160 size-table prefix)."""
    x = synth.generate(synth.CONFIGS["cesm"], slab=(0, 12)).numpy()
    s = orc.compress(x, "abs", 1e-3)
    for bad in (s[:-1], s + b"\0", b"XFPL" + s[4:]):
        with pytest.raises(cpu.PFPLCPUError) as e:
            cpu.decompress(bad)
        assert e.value.code == -4
    rng = np.random.default_rng(3)
    for _ in range(300):
        b = bytearray(s)
        i = int(rng.integers(48, len(b)))
        b[i] ^= 1 << int(rng.integers(0, 8))
        try:
            cpu.decompress(bytes(b))
        except cpu.PFPLCPUError as e:
            assert e.code == -4
