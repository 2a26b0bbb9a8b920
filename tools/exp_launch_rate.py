"""How many dependent kernel launches per second does the GPU retire across P independent chains?
One CUDA graph holding P parallel chains of tiny dependent kernels (captured with fork/join), replayed
once: no host launch cost inside the measurement."""
import torch

def main():
    K = 2000  # kernels per chain
    for P in (1, 2, 4, 8, 16):
        xs = [torch.zeros(64, device="cuda") for _ in range(P)]
        streams = [torch.cuda.Stream() for _ in range(P)]
        cap = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=cap):
            ev = torch.cuda.Event()
            ev.record(cap)
            for s in streams:
                s.wait_event(ev)
            for p in range(P):
                with torch.cuda.stream(streams[p]):
                    for _ in range(K):
                        xs[p].add_(1)
            for s in streams:
                e = torch.cuda.Event()
                e.record(s)
                cap.wait_event(e)
        g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3
        print(f"P={P}: {us / K:.2f} us per kernel per chain -> {P * K / us:.2f} M kernels/s total")

if __name__ == "__main__":
    main()
