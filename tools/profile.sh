#!/bin/bash
# ncu evidence for the current build (run on a GPU box from the repo root):
#   bash tools/profile.sh TAG
# 1. launch list of the bench command (per-launch gpu__time_duration, cold
#    cache, serialised -- the kernels' SHARE of a step, not a bench number);
# 2. one `--set full` capture of K1 (stream + fused report phase) on the bench workload (C4);
# 3. one `--set full` capture of K1 on C2A (Jacobi-2D 8192^2 fp32, clean).
set -u
TAG=${1:-prof}
OUT=gpurun_out
NCU=/usr/local/cuda/bin/ncu
$NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:arcv_ -c 40 --csv \
  --log-file $OUT/${TAG}_launches_c4.csv python bench.py --profile --steps 4 --warmup 3 > $OUT/${TAG}_launches_run.log 2>&1
echo "launches rc=$?"
$NCU --set full --clock-control none --import-source on -k regex:arcv_stream_kernel -s 3 -c 1 \
  -o $OUT/${TAG}_k1_c4 -f python bench.py --profile --steps 1 --warmup 3 > $OUT/${TAG}_k1_c4.log 2>&1
echo "k1 rc=$?"
$NCU --set full --clock-control none --import-source on -k regex:arcv_stream_kernel -s 3 -c 1 \
  -o $OUT/${TAG}_k1_c2a -f python -c "
import sys; sys.path.insert(0, '.')
import torch, synth, paper_conf_ipps_leelv14_b200 as av
av.init(0)
o, r = synth.C2('A').slice(device='cuda')
for _ in range(5): av.compare(o, r, 0.0, 1e-5, 1 << 20)
torch.cuda.synchronize(); av.finalize()
" > $OUT/${TAG}_k1_c2a.log 2>&1
echo "k1 c2a rc=$?"
# C2B (two dense tiles, pinned report: split + coalesced direct writes), C3 (one
# batched launch over twelve regions), C5 (int32 2^30, 50 % mismatches: group path)
for cfg in c2b c3 c5; do
$NCU --set full --clock-control none --import-source on -k regex:arcv_stream_kernel -s 3 -c 1 \
  -o $OUT/${TAG}_k1_$cfg -f python -c "
import sys; sys.path.insert(0, '.')
import torch, synth, paper_conf_ipps_leelv14_b200 as av
av.init(0)
cfg = '$cfg'
if cfg == 'c2b':
    o, r = synth.C2('B').slice(device='cuda')
    rep = torch.empty(24 << 20, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
    for _ in range(5): av.compare(o, r, 0.0, 1e-5, 1 << 20, report=rep)
elif cfg == 'c3':
    regs = synth.c3_regions()
    data = [rg.slice(device='cuda') for rg in regs]
    pb = av.prepare_batch([(o, r, rg.abs_tol, rg.rel_tol, rg.max_report, rg.name) for rg, (o, r) in zip(regs, data)])
    for _ in range(5): pb()
else:
    c5 = synth.C5()
    o, r = c5.slice(device='cuda')
    drep = torch.empty(24 << 20, dtype=torch.uint8, device='cuda')
    for _ in range(5): av.compare(o, r, 0, 0, 1 << 20, report=drep)
torch.cuda.synchronize(); av.finalize()
" > $OUT/${TAG}_k1_$cfg.log 2>&1
echo "k1 $cfg rc=$?"
done
for f in k1_c4 k1_c2a k1_c2b k1_c3 k1_c5; do
  $NCU -i $OUT/${TAG}_$f.ncu-rep --page raw --csv > $OUT/${TAG}_${f}_raw.csv 2>/dev/null
  $NCU -i $OUT/${TAG}_$f.ncu-rep --page details --csv > $OUT/${TAG}_${f}_details.csv 2>/dev/null
  # the .ncu-rep files are large (gpurun copies back <= 64 MiB): keep them only on request
  [ -n "${KEEP_REP:-}" ] || rm -f $OUT/${TAG}_$f.ncu-rep
done
echo done
