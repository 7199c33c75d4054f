OUT=gpurun_out/s2h; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_graphs.py tests/test_gpu_logical_devices.py tests/test_gpu_fullsize.py -x -q > $OUT/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest.log
NCU=1 bash tools/ab_tb2.sh s2h/ab main v3ml
