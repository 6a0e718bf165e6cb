"""Run tests/test_gpu_peer.py's two-process IPC worker with faulthandler output in
gpurun_out/ (debugging a crash)."""
import os
import socket
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def worker(rank, world, port, outdir):
    import faulthandler
    fh = open(os.path.join(outdir, "fh%d.txt" % rank), "w")
    faulthandler.enable(fh, all_threads=True)
    import test_gpu_peer
    test_gpu_peer._ipc_worker(rank, world, port, outdir)


if __name__ == "__main__":
    import torch.multiprocessing as mp
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    out = os.path.join(ROOT, "gpurun_out")
    os.makedirs(out, exist_ok=True)
    mp.start_processes(worker, args=(2, port, out), nprocs=2, join=True, start_method="spawn")
