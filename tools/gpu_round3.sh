mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/w_smoke.log 2>&1
timeout 2000 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/w_gpu_tests.log 2>&1
timeout 600 python bench.py > gpurun_out/w_bench.json 2> gpurun_out/w_bench.err
timeout 900 python bench.py --workload corr --no-cpu-baseline > gpurun_out/w_bench_corr.json 2>> gpurun_out/w_bench.err
timeout 900 python bench.py --workload contract --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/w_bench_contract.json 2>> gpurun_out/w_bench.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 300 --csv --log-file gpurun_out/w_launches_corr.csv python bench.py --workload corr --profile > gpurun_out/w_prof.log 2>&1
echo done
