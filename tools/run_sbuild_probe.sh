mkdir -p gpurun_out/sb2
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "S_" > gpurun_out/sb2/s_tests.txt 2>&1; echo "S tests rc=$?"; tail -3 gpurun_out/sb2/s_tests.txt
for V in 0 1; do CUALIGN_SBUILD_VAR=$V CUALIGN_INIT_TRACE=1 timeout 600 python tools/probe_init.py O 1.0 > gpurun_out/sb2/init_v$V.txt 2>&1; echo "var $V"; tail -13 gpurun_out/sb2/init_v$V.txt; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_sbuild_g --launch-count 2 -o gpurun_out/sb2/sbuild_g python tools/probe_init.py O 1.0 > gpurun_out/sb2/ncu.txt 2>&1; echo "ncu rc=$?"
