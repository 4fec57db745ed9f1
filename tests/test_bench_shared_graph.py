"""bench.py at N > 1 (CPU, gloo, world 2): the node's local rank 0 generates the CSR once into
shared files and both ranks map the same bytes; the files are removed at the end. Keeps host RAM at
one graph copy whatever N is (C4: 26 GB, C5: 72 GB on a 196 GB box)."""
import os
import socket
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import hashlib, os, sys, glob
sys.path.insert(0, %(root)r)
import numpy as np
import torch.distributed as dist
dist.init_process_group("gloo")
import bench, graphgen as gg
rank = dist.get_rank()
os.environ["ASCETIC_SHM_DIR"] = %(tmp)r
g, cleanup, gen_s = bench.shared_graph("c1", dist.barrier, int(os.environ["LOCAL_RANK"]), "t%(port)d")
ref = gg.config_graph("c1")
assert g.n == ref.n and g.m == ref.m and not g.pairs
assert np.array_equal(g.off, ref.off) and np.array_equal(g.nbr, ref.nbr)
assert (gen_s > 0) == (rank == 0)                       # generated once, by local rank 0
h = hashlib.sha1(np.asarray(g.nbr).tobytes()).hexdigest()
print("rank", rank, "ok", h, flush=True)
del g
cleanup()
dist.barrier()
left = glob.glob("/dev/shm/ascetic_c1_t%(port)d*") + glob.glob(os.path.join(%(tmp)r, "ascetic_c1_t%(port)d*"))
assert not left, left
dist.destroy_process_group()
"""


def test_shared_graph_world2(tmp_path):
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    script = tmp_path / "sg.py"
    script.write_text(SCRIPT % {"root": ROOT, "tmp": str(tmp_path), "port": port})
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", str(port), str(script)],
                       cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-3000:]
    hashes = {line.split()[3] for line in r.stdout.splitlines() if line.startswith("rank")}
    assert len(hashes) == 1
