OUT=gpurun_out/s2j; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_graphs.py tests/test_gpu_logical_devices.py tests/test_gpu_fullsize.py -x -q > $OUT/pytest.log 2>&1; echo "pytest rc=$?"; tail -5 $OUT/pytest.log
SOMIER_LIB=$PWD/paper_conf_ipps_torresft22_b200/libsomier_kw11.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "TB2 or 4" > $OUT/pytest_kw11.log 2>&1; echo "pytest kw11 rc=$?"; tail -2 $OUT/pytest_kw11.log
NCU=1 bash tools/ab_tb2.sh s2j/ab main v3ml kw11
