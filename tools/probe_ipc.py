"""Probe: CUDA IPC between two processes on the same GPU (used by the dist tests)."""
import multiprocessing as mp
import sys

import torch


def child(q_in, q_out):
    from cuda.bindings import runtime as rt
    torch.cuda.set_device(0)
    h = q_in.get()
    handle = rt.cudaIpcMemHandle_t()
    handle.reserved = h
    err, ptr = rt.cudaIpcOpenMemHandle(handle, rt.cudaIpcMemLazyEnablePeerAccess)
    if err != rt.cudaError_t.cudaSuccess:
        q_out.put(f"open failed {err}")
        return
    # write 42 into the parent's buffer through the mapped pointer
    err, = rt.cudaMemset(ptr, 42, 16)
    torch.cuda.synchronize()
    q_out.put(f"child ok err={err}")
    rt.cudaIpcCloseMemHandle(ptr)


def main():
    from cuda.bindings import runtime as rt
    ctx = mp.get_context("spawn")
    q_in, q_out = ctx.Queue(), ctx.Queue()
    p = ctx.Process(target=child, args=(q_in, q_out))
    p.start()
    torch.cuda.set_device(0)
    t = torch.zeros(64, dtype=torch.uint8, device="cuda")
    err, h = rt.cudaIpcGetMemHandle(t.data_ptr())
    print("get handle", err)
    q_in.put(bytes(h.reserved))
    print(q_out.get(timeout=120))
    p.join(timeout=60)
    print("parent sees", t[:16].tolist())
    sys.exit(0 if t[0].item() == 42 else 1)


if __name__ == "__main__":
    main()
