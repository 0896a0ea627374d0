"""One rank of tests/test_gpu_configs.py::test_two_process_ipc_gather (not a
test module): two processes on cuda:0, gloo (file rendezvous) for the
barrier and the handle exchange; rank 0 owns the break map, rank 1 maps it
through CUDA IPC and its kernel writes its shard straight into it.

  python tests/_ipc_worker.py RANK WORLD INIT_FILE OUT_NPZ
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icde_giesekerhvo20_b200 import binding, synth  # noqa: E402


def main():
    rank, world, init_file, out_npz = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3], sys.argv[4]
    dist.init_process_group("gloo", init_method=f"file://{init_file}", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    spec = synth.StackSpec(P=300_000, N=230, n_hist=115, miss=0.6, mask="cloud", seed=17)
    b, e = binding.shard_range(spec.P, rank, world)
    Y, dates = synth.generate(spec, "cuda:0", columns=(b, e))
    plan = binding.Plan(0, spec.N, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    if rank == 0:
        brk = torch.full((spec.P,), -7, dtype=torch.int32, device="cuda:0")
        mag = torch.full((spec.P,), float("nan"), dtype=torch.float32, device="cuda:0")
        handles = [binding.ipc_export(brk), binding.ipc_export(mag)]
    else:
        handles = [None, None]
    dist.broadcast_object_list(handles, src=0)
    if rank == 0:
        pb, pm = brk.data_ptr(), mag.data_ptr()
    else:
        pb, pm = binding.ipc_open(handles[0], 0), binding.ipc_open(handles[1], 0)
    # this rank's slice of the map: the epilogue stores land in rank 0's memory
    plan.execute(Y, out={"break": pb + 4 * b, "magnitude": pm + 4 * b}, check_out=False)
    torch.cuda.synchronize()
    dist.barrier()
    if rank == 0:
        np.savez(out_npz, brk=brk.cpu().numpy(), mag=mag.cpu().numpy())
    dist.barrier()
    if rank != 0:
        binding.ipc_close(pb)
        binding.ipc_close(pm)
    plan.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
