mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v_smoke.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/v_gpu_tests.log 2>&1
timeout 600 python bench.py > gpurun_out/v_bench.json 2> gpurun_out/v_bench.err
timeout 900 python bench.py --workload corr --no-cpu-baseline > gpurun_out/v_bench_corr.json 2>> gpurun_out/v_bench.err
timeout 900 python bench.py --workload contract --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/v_bench_contract.json 2>> gpurun_out/v_bench.err
echo done
