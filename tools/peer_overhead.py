"""Cost of the in-kernel cross-GPU combine on one GPU.

cfg4b column sum [65536,1024] f16 -> f32, timed with CUDA events over
back-to-back launches on rotating input copies (> L2):
  plain      fop_run, no exchange (default geometry, tuning off)
  peer W=1   fop_run_peer with a group of one: the epilogue's epoch bump,
             push, release flag, acquire wait and combine all run, against
             the rank's own buffer
  nccl-less  the NCCL baseline cannot run on one GPU; its cost on a real
             node is one extra kernel + a 4 KiB all-reduce per step

    python tools/peer_overhead.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import torch  # noqa: E402

import workloads as W  # noqa: E402
from harness import device_tensors  # noqa: E402
from paper_conf_cgo_bastoulzrlsjfjc22_b200 import FusedOp, PeerGroup  # noqa: E402


def timeit(fn, copies, reps=200):
    for k in range(10):
        fn(copies[k % len(copies)])
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for k in range(reps):
        fn(copies[k % len(copies)])
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) / reps * 1e3


def main():
    desc = W.cfg4b()
    x = W.make_inputs(desc)
    copies = [device_tensors(desc, x) for _ in range(3)]
    nbytes = W.algorithmic_bytes(desc)
    res = {}
    plain = FusedOp(desc, autotune=0)
    res["plain_us"] = timeit(lambda t: plain.run(t), copies)
    peer = FusedOp(desc, autotune=0, peer_world=1, peer_loop="r")
    buf = torch.zeros(peer.peer_bytes, dtype=torch.uint8, device="cuda")
    g = PeerGroup(0, [buf.data_ptr()])
    res["peer_w1_us"] = timeit(lambda t: peer.run(t, peers=g), copies)
    res["peer_err"] = int(buf[-16:].view(torch.int32)[0])
    # same results: the combine of one rank adds its sums to +0 in order
    peer.run(copies[0], peers=g)
    torch.cuda.synchronize()
    b = copies[0]["out"].clone()
    plain.run(copies[0])
    torch.cuda.synchronize()
    res["identical_to_plain"] = bool(torch.equal(copies[0]["out"].view(torch.int32), b.view(torch.int32)))
    res["GBs_plain"] = nbytes / res["plain_us"] / 1e3
    res["GBs_peer_w1"] = nbytes / res["peer_w1_us"] / 1e3
    print(json.dumps(res))


if __name__ == "__main__":
    main()
