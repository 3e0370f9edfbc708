#!/bin/bash
# Copy the summaries of a tools/_gpu_measure.sh pass (gpurun_out/) into profiles/ under round tag R (default r2).
R=${R:-r2}
G=gpurun_out
P=profiles
last() { tail -1 "$1"; }
last $G/bench.log > $P/bench_$R.json
last $G/bench_sync.log > $P/bench_sync_$R.json
last $G/bench_cfg5.log > $P/bench_cfg5_$R.json
last $G/bench_cfg1.log > $P/bench_cfg1_$R.json
last $G/bench_ref.log > $P/bench_ref_$R.json
cp $G/launches.csv $P/launches_bench_$R.csv
cp $G/launches.txt $P/launches_bench_$R.txt
cp $G/ncu_full.txt $P/ncu_full_$R.txt
cp $G/ncu_summary.json $P/ncu_summary_$R.json
cp $G/ncu_summary.json $P/ncu_summary.json
cp $G/ncu_details.csv.gz $P/ncu_details_$R.csv.gz
mkdir -p $P/ncu_configs_$R
cp $G/ncu_cfg*.json $G/ncu_cfg*.txt $P/ncu_configs_$R/
cp $G/sweep.json $P/sweep_$R.json
cp $G/variants.json $P/variants_$R.json
cp $G/methods.json $P/methods_$R.json
cp $G/oracle_time.json $P/oracle_time_$R.json
cp $G/pipeline.txt $P/pipeline_$R.txt
cp $G/trace_kernels.txt $P/trace_kernels_$R.txt
cp $G/trace_view.txt $P/trace_tiles_$R.txt
# sanitizer logs only from a pass where compute-sanitizer ran (the pool closed it late in round 2)
if ! grep -q "is closed on this pool" $G/sanitize_memcheck.log 2>/dev/null; then
  mkdir -p $P/sanitize_$R
  cp $G/sanitize_memcheck.log $G/sanitize_racecheck.log $G/sanitize_synccheck.log $P/sanitize_$R/
fi
cp $G/rand_probe.txt $P/rand_probe_$R.txt
