mkdir -p gpurun_out
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/l_f64.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_f64.py tests/test_gpu_apps.py tests/test_gpu_shard.py tests/test_gpu_fullsize.py tests/test_gpu_studies.py -m gpu -q -x -p no:cacheprovider > gpurun_out/l_tests.log 2>&1
timeout 900 python bench.py --workload corr --no-cpu-baseline > gpurun_out/l_bench_corr.json 2> gpurun_out/l_bench.err
timeout 600 ncu --set full --clock-control none -k regex:gemm_dmma_kernel -c 1 -o /tmp/l_dmma python tools/f64_probe.py 8192 > gpurun_out/l_ncu.log 2>&1
ncu -i /tmp/l_dmma.ncu-rep --page details --csv > gpurun_out/l_dmma_details.csv 2>/dev/null
ncu -i /tmp/l_dmma.ncu-rep --page raw --csv > gpurun_out/l_dmma_raw.csv 2>/dev/null
timeout 600 ncu --set full --clock-control none -k regex:gemm_ffma_kernel -c 1 -o /tmp/l_ffma python tools/f32_probe.py 8192 > gpurun_out/l_ncu2.log 2>&1
ncu -i /tmp/l_ffma.ncu-rep --page details --csv > gpurun_out/l_ffma_details.csv 2>/dev/null
ncu -i /tmp/l_ffma.ncu-rep --page raw --csv > gpurun_out/l_ffma_raw.csv 2>/dev/null
rm -f /tmp/l_dmma.ncu-rep /tmp/l_ffma.ncu-rep
echo done
