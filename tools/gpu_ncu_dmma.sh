mkdir -p gpurun_out
timeout 600 python tools/f64_probe.py 8192 > gpurun_out/m_f64.txt 2>&1
timeout 600 ncu --set full --clock-control none -k regex:gemm_dmma_kernel -c 1 -o /tmp/m_dmma python tools/f64_probe.py 8192 > gpurun_out/m_ncu.log 2>&1
ncu -i /tmp/m_dmma.ncu-rep --page raw --csv > gpurun_out/m_dmma_raw.csv 2>/dev/null
ncu -i /tmp/m_dmma.ncu-rep --page details --csv > gpurun_out/m_dmma_details.csv 2>/dev/null
rm -f /tmp/m_dmma.ncu-rep
timeout 900 python -m pytest tests/test_gpu_f64.py tests/test_gpu_smoke*.py -m gpu -q -x -p no:cacheprovider > gpurun_out/m_tests.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/m_smoke.log 2>&1
echo done
