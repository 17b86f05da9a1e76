#!/bin/bash
# Round-2 validation on one B200: smoke, GPU tests, default bench (cfg2 + cfg3/4/5 secondaries),
# the torchrun branch as a 2-rank gloo dry run sharing the GPU, the reference arm.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout ${PYT:-1800} python -m pytest tests -q -m gpu -x ${PYARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for w in cfg5 cfg4; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus 2 --steps 3 --warmup 3 --workload $w --backend gloo > gpurun_out/bench_gloo2_$w.json 2> gpurun_out/bench_gloo2_$w.err
done
timeout 300 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
rm -rf gpurun_out/jitc
