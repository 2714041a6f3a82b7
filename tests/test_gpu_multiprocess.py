"""The cross-process data plane on ONE GPU: two processes, one rank each, joined by the host
transport (memxct_plan_set_comm_host: a shared-memory rendezvous, CUDA-IPC device mailboxes
for the collectives).  With EXCHANGE = 1 the SpMV epilogue and the pack kernel store straight
into the OTHER PROCESS's buffers through cudaIpcOpenMemHandle mappings, and the epoch / credit
flags are system-scope stores and acquire loads across the process boundary -- the NVLink path of
P:744-756 minus the link.  (NCCL cannot be used here: it rejects two ranks on one device.)

Every output -- repeated forwards and backs (credits), a 10- and a 30-iteration CGLS with
residuals -- is bit-identical to the same 2-rank decomposition on virtual ranks in one process
(tests/test_gpu_multirank.py), for the sparse all-to-allv, the dense reduce-scatter / allgather
and the fused peer exchange (one-thread waits, the default when ranks share a GPU, and the folded
waits inside the data kernels that NCCL ranks use, MEMXCT_PEER_FOLD=1)."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

from paper_conf_sc_hidayetoglubgrg19_b200 import inputs
from test_gpu_multirank import build_group, run_ranks, scatter

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_hidayetoglubgrg19_b200 import build_ext
    build_ext.build()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def run_processes(out_dir, exchange, geom, nranks=2, extra_env=None, timeout=600):
    port = _free_port()
    procs = []
    for r in range(nranks):
        env = dict(os.environ, RANK=str(r), WORLD_SIZE=str(nranks), MASTER_ADDR="127.0.0.1",
                   MASTER_PORT=str(port), CUDA_MODULE_LOADING="EAGER", **(extra_env or {}))
        procs.append(subprocess.Popen([sys.executable, os.path.join(HERE, "proc_cases.py"), str(out_dir),
                                       exchange, *map(str, geom)], env=env, stdout=subprocess.PIPE,
                                      stderr=subprocess.PIPE, text=True))
    outs = []
    for p in procs:
        try:
            o, e = p.communicate(timeout=timeout)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        outs.append((p.returncode, o, e))
    for rc, o, e in outs:
        assert rc == 0 and "CASE OK" in o, (rc, o[-2000:], e[-4000:])
    return [dict(np.load(os.path.join(out_dir, f"rank{r}.npz"))) for r in range(nranks)]


_REF = {}


def virtual_reference(geom, nranks=2):
    """The same sequence on virtual ranks (collective exchange), per rank."""
    key = (geom, nranks)
    if key in _REF:
        return _REF[key]
    n, m, c = geom
    _, plans = build_group(n, m, c, nranks)
    xs = scatter(plans, inputs.uniform(n * n, 1), 0, np.float32)
    ys = scatter(plans, inputs.uniform(m * c, 2), 1, np.float32)

    def body(r):
        p, x, y = plans[r], xs[r], ys[r]
        o = {"f1": p.forward(x), "f2": p.forward(2 * x), "b1": p.back(y), "b3": p.back(3 * y),
             "f1b": p.forward(x), "b1b": p.back(y)}
        o["cg10"], o["r10"] = p.cg(y, 10, residuals=True)
        o["cg30"], o["r30"] = p.cg(y, 30, residuals=True)
        o["pix"], o["ray"] = p.local_indices(0), p.local_indices(1)
        return {k: (v.cpu().numpy() if hasattr(v, "cpu") else v) for k, v in o.items()}
    _REF[key] = run_ranks(nranks, body)
    for p in plans:
        p.close()
    return _REF[key]


CASES = [("collective", None), ("dense", None), ("peer", None), ("peer", {"MEMXCT_PEER_FOLD": "1"})]


@pytest.mark.parametrize("exchange,env", CASES, ids=["collective", "dense", "peer", "peer-folded"])
@pytest.mark.parametrize("geom", [(64, 90, 64), (256, 360, 256)])
def test_two_processes_one_gpu_bit_identical_to_virtual_ranks(tmp_path, exchange, env, geom):
    got = run_processes(tmp_path, exchange, geom, extra_env=env)
    ref = virtual_reference(geom)
    for r in range(2):
        assert np.array_equal(got[r]["pix"], ref[r]["pix"]) and np.array_equal(got[r]["ray"], ref[r]["ray"])
        for k in ("f1", "f2", "b1", "b3", "f1b", "b1b", "cg10", "cg30", "r10", "r30"):
            assert np.array_equal(got[r][k], ref[r][k]), (r, k)
    assert got[0]["sent"] > 0 and got[0]["peers"] == 1      # data really crossed the process boundary
