# GPU validation: full pytest -m gpu, smoke, C2 bench line (used through gpurun; writes gpurun_out/)
mkdir -p gpurun_out
TAG=${1:-run}
timeout 1500 python -m pytest tests -m gpu -x -q --durations=8 --timeout 400 > gpurun_out/gpu_tests_$TAG.log 2>&1; echo "gpu tests rc=$?" >> gpurun_out/gpu_tests_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_c2_$TAG.json 2> gpurun_out/bench_c2_$TAG.err
