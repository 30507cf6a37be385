"""f2 measurement: FastID-1M shape (64 queries x 1M x 4096 SNPs, XOR + ANDNOT best) with the
packed database (and its popcounts) in pinned HOST memory, streamed through two device
buffers (paper's end-to-end mode).  Reports comparisons/s end to end and the
H2D rate achieved, next to a plain pageable-free H2D copy of the same bytes."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_binderlp19_b200 as snp
from paper_conf_ipps_binderlp19_b200.stream import stream_search
torch.cuda.set_device(0)
nq, nd, nbits = 64, 1_000_000, 4096
w = snp.snp_words(nbits)
Dd = torch.randint(-2**62, 2**62, (nd, w), dtype=torch.int64, device="cuda").view(torch.uint64)
pd = snp.snp_row_popc(Dd, nbits)
D_host = Dd.cpu().pin_memory(); P_host = pd.cpu().pin_memory()
Q = torch.randint(-2**62, 2**62, (nq, w), dtype=torch.int64, device="cuda").view(torch.uint64)
def t(fn, reps=5):
    fn(); torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps
out = {}
buf = torch.empty_like(Dd)
out["h2d_only_ms"] = t(lambda: buf.copy_(D_host, non_blocking=True))
for ch in (1 << 17, 1 << 18, 1 << 19):
    out[f"stream_ms_chunk{ch}"] = t(lambda: stream_search(Q, D_host, nbits, ("xor", "andnot"), popD_host=P_host, chunk_rows=ch))
best = min(v for k, v in out.items() if k.startswith("stream"))
out["bytes"] = nd * w * 8 + nd * 4
out["h2d_GBps"] = out["bytes"] / (out["h2d_only_ms"] / 1e3) / 1e9
out["stream_cmp_per_s"] = 2 * nq * nd * nbits / (best / 1e3)
out["resident_step_ms_ref"] = t(lambda: snp.snp_fastid_search(Q, Dd, nbits, ("xor", "andnot"), counts=False, popD=pd))
print(json.dumps(out))
