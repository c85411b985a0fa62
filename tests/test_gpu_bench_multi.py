"""bench.py's N>1 path on ONE GPU: two ranks under torchrun share cuda:0 over gloo (the test
hooks BENCH_GPU_INDEX / BENCH_DIST_BACKEND; the driver's runs use one GPU per rank and NCCL).  Exercises the real
kernels behind the sharded mode: rank 0 scatters the shards (sharded.py), per-rank compact B rows, the timed SpMM
with max over ranks, the exchange timings and the column-chunk pipeline (spmm_run_ld), whose C must be
bit-identical to the plain run."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("exchange,ranks", [("rows", 2), ("broadcast", 2), ("rows", 3)])
def test_bench_ranks_one_gpu(exchange, ranks):
    env = {**os.environ, "BENCH_GPU_INDEX": "0", "BENCH_DIST_BACKEND": "gloo"}
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(ranks), "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"), "--gpus", str(ranks), "--config", "c1",
           "--steps", "3", "--warmup", "3", "--policy-steps", "2", "--e2e-steps", "3", "--no-cpu-baseline",
           "--no-cusparse", "--b-exchange", exchange, "--policies", "identity,nnz_sort,cta_aware"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == ranks and d["value"] > 0 and d["gpu_launches"] > 0
    m = d["multi_gpu"]
    assert m["b_exchange"]["ms"] > 0 and m["c_allgather"]["ms"] > 0 and m["spmm_ms"] > 0
    if exchange == "rows":
        assert m["pipelined"]["bit_identical_to_run"] is True
        assert m["b_alltoall"]["equals_distribute_B"] is True and m["b_alltoall"]["ms"] > 0
        assert d["e2e"]["h2d_bytes_per_step"] < d["config"]["N"] * d["config"]["K"] * 4 * 2
