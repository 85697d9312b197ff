#!/bin/bash
# Warp-stall sampling of K1 on small, tail-dominated calls (C1; C4 at 2^26 =
# the p = 8 shard): where the fixed cost per call goes.  Exports the details
# page (WarpStateStats: stall reasons, incl. "No Instruction" = i-cache misses)
# and the per-SASS-line source page with sampled stall reasons.
#   bash tools/profile_stalls.sh TAG
set -u
TAG=${1:-stalls}
OUT=gpurun_out
NCU=/usr/local/cuda/bin/ncu
for cfg in c1 c4s; do
$NCU --set full --import-source on --clock-control none -k regex:arcv_stream_kernel -s 4 -c 1 \
  -o $OUT/${TAG}_$cfg -f python -c "
import sys; sys.path.insert(0, '.')
import torch, synth, paper_conf_ipps_leelv14_b200 as av
av.init(0)
rep = torch.empty(24 << 20, dtype=torch.uint8, pin_memory=True).numpy().view(av.REPORT_DTYPE)
c = synth.C1() if '$cfg' == 'c1' else synth.C4(1 << 26)
o, r = c.slice(device='cuda')
for _ in range(6): av.compare(o, r, c.abs_tol, c.rel_tol, c.max_report, report=rep)
torch.cuda.synchronize(); av.finalize()
" > $OUT/${TAG}_$cfg.log 2>&1
echo "$cfg rc=$?"
$NCU -i $OUT/${TAG}_$cfg.ncu-rep --page details --csv > $OUT/${TAG}_${cfg}_details.csv 2>/dev/null
$NCU -i $OUT/${TAG}_$cfg.ncu-rep --page raw --csv > $OUT/${TAG}_${cfg}_raw.csv 2>/dev/null
$NCU -i $OUT/${TAG}_$cfg.ncu-rep --page source --csv --print-source sass > $OUT/${TAG}_${cfg}_source_sass.csv 2>/dev/null
[ -n "${KEEP_REP:-}" ] || rm -f $OUT/${TAG}_$cfg.ncu-rep
done
gzip -f $OUT/${TAG}_*_source_sass.csv
ls -la $OUT/${TAG}_*
