"""Fused peer-memory exchange (EXCHANGE = 1) on virtual ranks: the SpMV
epilogue stores partials into the owners' receive buffers and the pack kernel stores ray values
into the peers' footprint buffers, synchronised by epoch / credit flags.  The reductions read the
same partials in the same peer order as the collective path, so results must be bit-identical to
EXCHANGE = 0 for any call sequence (including repeated forwards, which exercise the credits).
Each case runs in a child process (tests/peer_cases.py explains why)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext
    build_ext.build()


def run_case(*args):
    r = subprocess.run([sys.executable, os.path.join(HERE, "peer_cases.py"), *map(str, args)],
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "CASE OK" in r.stdout, (r.stdout[-2000:], r.stderr[-4000:])


@pytest.mark.parametrize("nranks", [1, 2, 3, 4])
@pytest.mark.parametrize("geom", [(64, 90, 64), (256, 360, 256)])
def test_peer_exchange_bit_identical_to_collective(nranks, geom):
    run_case("projections", nranks, *geom)


def test_peer_exchange_cg():
    run_case("cg", 4, 256, 360, 256)


@pytest.mark.parametrize("ray_block", [2, 8])
def test_peer_exchange_blocked_rows(ray_block):
    """Forward rows grouped in projection blocks (RAY_BLOCK): the fused epilogue stores each
    partial at its footprint position, so outputs stay bit-identical to the collective path on
    Hilbert rows."""
    run_case("projections", 3, 256, 360, 256, ray_block)
