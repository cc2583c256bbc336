mkdir -p gpurun_out
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/j_f64.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_f64.py tests/test_gpu_apps.py tests/test_gpu_faults.py tests/test_gpu_shard.py tests/test_gpu_fullsize.py tests/test_gpu_sanitizer.py -m gpu -q -x -p no:cacheprovider > gpurun_out/j_tests.log 2>&1
timeout 900 python bench.py --workload corr --no-cpu-baseline > gpurun_out/j_bench_corr.json 2> gpurun_out/j_bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_dmma_kernel -c 1 -o gpurun_out/j_dmma python tools/f64_probe.py 8192 > gpurun_out/j_ncu.log 2>&1
echo done
