"""H2D copy rate of a 1-GiB pinned buffer (the e2e leg of bench.py is bound by it): one
cudaMemcpyAsync on one stream vs the same bytes split over 2 / 4 streams, and the rate
while nothing else runs. Diagnostic only."""
import torch

B = 1 << 30
h = torch.empty(B, dtype=torch.uint8).pin_memory()
h.fill_(7)
d = torch.empty(B, dtype=torch.uint8, device="cuda")
streams = [torch.cuda.Stream() for _ in range(8)]
main = torch.cuda.current_stream()


def run(nsplit, piece_mb=None):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(main)
    piece = B // nsplit if piece_mb is None else piece_mb << 20
    ends = []
    for i, off in enumerate(range(0, B, piece)):
        s = streams[i % nsplit]
        s.wait_event(e0)
        with torch.cuda.stream(s):
            d[off:off + piece].copy_(h[off:off + piece], non_blocking=True)
            ev = torch.cuda.Event()
            ev.record(s)
        ends.append(ev)
    for ev in ends:
        main.wait_event(ev)
    e1.record(main)
    torch.cuda.synchronize()
    return B / (e0.elapsed_time(e1) / 1e3) / 1e9


for rep in range(2):
    for ns in (1, 2, 4, 8):
        print(f"H2D 1 GiB over {ns} stream(s): {run(ns):.1f} GB/s", flush=True)
    for mb in (8, 32, 128):
        print(f"H2D 1 GiB in {mb}-MiB pieces over 2 streams: {run(2, mb):.1f} GB/s", flush=True)
