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
for f in k1_c4 k1_c2a; do
  $NCU -i $OUT/${TAG}_$f.ncu-rep --page raw --csv > $OUT/${TAG}_${f}_raw.csv 2>/dev/null
  $NCU -i $OUT/${TAG}_$f.ncu-rep --page details --csv > $OUT/${TAG}_${f}_details.csv 2>/dev/null
done
echo done
