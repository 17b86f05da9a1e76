cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --workload cfg2 --steps 20 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err
python tools/stage_times.py 2 3 > gpurun_out/stages.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_cfg2.csv python bench.py --workload cfg2 --steps 2 --warmup 3 --no-cpu-baseline --no-secondary > /dev/null 2>&1
