mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/t_smi.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/t_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/t_gpu_tests.log 2>&1
timeout 600 python bench.py > gpurun_out/t_bench.json 2> gpurun_out/t_bench.err
timeout 600 python bench.py --workload corr --no-cpu-baseline > gpurun_out/t_bench_corr.json 2>> gpurun_out/t_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 900 --csv --log-file gpurun_out/t_launches.csv python bench.py --profile > gpurun_out/t_prof.log 2>&1
echo done
