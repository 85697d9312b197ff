"""Diagnostic: small mixed workload for compute-sanitizer (tools/sanitize.sh)."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth, oracle
import paper_conf_ipps_leelv14_b200 as av
av.init(0)
c1 = synth.C1(); o, r = c1.slice(0, 1 << 16); o, r = o.cuda(), r.cuda()
g = av.compare(o, r, 1e-6, 1e-5, 100); print("c1", g.n_mismatch)
g = av.compare(o[3:40003], r[1:40001], 1e-6, 1e-5, 10); print("mis", g.n_mismatch)
o5, r5 = synth.C5(1 << 18).slice(device="cuda")
g = av.compare(o5, r5, 0, 0, 5000); print("c5 group", g.n_mismatch)
regs = [(o[:1000], r[:1000], 1e-6, 1e-5, 5), (o5[:7777], r5[:7777], 0, 0, 9), (o.view(torch.uint8)[:333], r.view(torch.uint8)[:333], 0, 0, 4)]
res = av.batch(regs); print("batch", [x.n_mismatch for x in res])
g = av.compare(o.cpu().pin_memory(), r, 1e-6, 1e-5, 50); print("host", g.n_mismatch)
# round 2 paths: dense tiles split across CTAs with staged coalesced writes into a
# pinned / pageable / device report, a clean call (early, unfenced publish), count-only,
# the checksum screen between compares
od, rd = o[:4096 * 6].clone(), r[:4096 * 6].clone()
od[4096:8192] = rd[4096:8192] * 1.5 + 0.25
pin = torch.empty(24 * 20000, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
for rep in (pin, None, torch.empty(24 * 20000, dtype=torch.uint8, device="cuda")):
    g = av.compare(od, rd, 1e-6, 1e-5, 20000, report=rep); print("dense", g.n_mismatch)
g = av.compare(o, o, 1e-6, 1e-5, 100); print("clean", g.n_mismatch)
g = av.compare(o, r, 1e-6, 1e-5, 0); print("count-only", g.n_mismatch)
print("checksum", av.checksum(o)); g = av.compare(o, r, 1e-6, 1e-5, 100); print("after checksum", g.n_mismatch)
av.finalize()
print("SANITIZE-DONE")
