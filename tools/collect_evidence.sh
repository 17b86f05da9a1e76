#!/bin/bash
# Copy the summaries of a tools/gpu_final.sh run (gpurun_out/) into profiles/ under the round
# prefix: python-free, names as DESIGN.md / bench.py cite them.  Usage: tools/collect_evidence.sh r02
set -e
R=${1:?round prefix, e.g. r02}
cd "$(dirname "$0")/.."
G=gpurun_out
P=profiles
cp $G/bench_default.json $P/${R}_bench_cfg2.json
for w in cfg1 cfg3 cfg4 cfg5; do [ -s $G/bench_$w.json ] && cp $G/bench_$w.json $P/${R}_bench_$w.json; done
[ -s $G/bench_ref.json ] && cp $G/bench_ref.json $P/${R}_bench_reference_cfg2.json
for w in cfg2 cfg3 cfg4 cfg5; do [ -s $G/launches_$w.json ] && cp $G/launches_$w.json $P/${R}_launches_$w.json; done
cp_pair() { [ -s $G/$1.json ] && cp $G/$1.json $P/${R}_ncu_full_$2.json; [ -s $G/$1.regions.txt ] && cp $G/$1.regions.txt $P/${R}_ncu_regions_$2.txt; true; }
cp_pair prof_cfg2 tc_cfg2
cp_pair prof_cfg5 tc_cfg5
cp_pair prof_piv3 piv_cfg3
cp_pair prof_piv4 ptc_cfg4
cp_pair prof_piv4b ptc_border_cfg4
cp_pair prof_piv4cc piv_cfg4
tail -n 5 $G/pytest_gpu.log > $P/${R}_pytest_gpu.log
cp $G/smoke.log $P/${R}_smoke.log
for f in timeline_cfg2 timeline_cfg5; do [ -s $G/$f.txt ] && cp $G/$f.txt $P/${R}_$f.txt; done
[ -s $G/tc_prof2.json ] && cp $G/tc_prof2.json $P/${R}_tc_prof_cfg2.json
[ -s $G/piv_tc_prof4.json ] && cp $G/piv_tc_prof4.json $P/${R}_piv_tc_prof_cfg4.json
cat $G/tc_error5s.jsonl $G/tc_error2u.jsonl > $P/${R}_tc_error.jsonl 2>/dev/null || true
[ -s $G/umma_rates.log ] && cp $G/umma_rates.log $P/${R}_umma_rates.log
python tools/traffic_json.py $R $G
echo "collected into $P/${R}_*"
