cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 900 -p no:cacheprovider -k "packed_maps or exception_plans or enum_four or delta_rows or c4_auto" > gpurun_out/t2_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t2_pytest.log
