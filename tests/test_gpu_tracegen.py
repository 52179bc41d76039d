"""The device trace generator (tracegen/gen.cu) reproduces the host generator
(tracegen/records.py) bit for bit, so the full-size C3-C5 traces that bench.py
generates in HBM are the same traces the oracle-checked host path draws.

Chunks are taken at random offsets (straddling burst boundaries), at the first
and last records of the trace, and across every burst pattern (AFFINE sweeps,
RANDOM gathers, RANGE memcpy/memset records, RAW injected odd records).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from tracegen import build_config, build_tiny, gen_records  # noqa: E402
from tracegen.layout import PAT_AFFINE, PAT_RANDOM, PAT_RANGE, PAT_RAW  # noqa: E402


def _check(prog, i0, i1, dp):
    host = gen_records(prog, i0, i1)
    dev = dp.gen(i0, i1).cpu().numpy().view(host.dtype)
    assert np.array_equal(host.view(np.uint8), dev.view(np.uint8)), (prog.name, i0, i1)


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_device_generator_matches_host(name):
    from tracegen.device import DeviceProgram
    prog = build_config(name)
    dp = DeviceProgram(prog)
    n = prog.n_records
    rng = np.random.default_rng(7)
    chunk = 1 << 18
    starts = [0, max(0, n - chunk)] + [int(x) for x in rng.integers(0, n - chunk, 6)]
    # chunks that begin at burst starts of every pattern present
    for pat in (PAT_AFFINE, PAT_RANDOM, PAT_RANGE, PAT_RAW):
        idx = np.flatnonzero(prog.bursts["pattern"] == pat)
        if idx.size:
            b = int(idx[int(rng.integers(0, idx.size))])
            starts.append(max(0, min(int(prog.prefix[b]) - 7, n - chunk)))
    for i0 in starts:
        _check(prog, i0, i0 + chunk, dp)
    torch.cuda.synchronize()


def test_device_generator_tiny_programs():
    from tracegen.device import DeviceProgram
    for seed in range(20):
        prog = build_tiny(seed)
        dp = DeviceProgram(prog)
        _check(prog, 0, prog.n_records, dp)
        if prog.n_records > 3:
            _check(prog, 1, prog.n_records - 1, dp)
