#!/bin/bash
# The evidence set for one build (run on a GPU box from the repo root):
#   bash tools/final_evidence.sh TAG
# GPU tests + smoke, bench (ours and the reference arm), ncu launch list and
# --set full captures (tools/profile.sh), per-config and size-sweep
# timings.  Everything lands in gpurun_out/TAG_*.
set -u
TAG=${1:-final}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit,temperature.gpu --format=csv > $OUT/${TAG}_smi.txt
lscpu > $OUT/${TAG}_lscpu.txt
timeout 1500 python -m pytest tests -m gpu -q > $OUT/${TAG}_pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> $OUT/${TAG}_pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/${TAG}_smoke.txt 2>&1; echo "smoke rc=$?" >> $OUT/${TAG}_smoke.txt
python bench.py > $OUT/${TAG}_bench_c4.json 2> $OUT/${TAG}_bench_c4.err
python bench.py --impl reference > $OUT/${TAG}_bench_reference.json 2> $OUT/${TAG}_bench_reference.err
python tools/configs_perf.py > $OUT/${TAG}_configs_perf.log 2>&1
python tools/size_sweep.py f64 > $OUT/${TAG}_size_sweep_f64.log 2>&1
bash tools/profile.sh $TAG > $OUT/${TAG}_profile.log 2>&1
python tools/ncu_summary.py $TAG > $OUT/${TAG}_ncu_summary.json 2> $OUT/${TAG}_ncu_summary.err
# compute-sanitizer (tools/sanitize.sh) is closed on this GPU pool since round 2's last
# session; the last sanitizer evidence is profiles/r02final2_sanitizers.txt
echo done
