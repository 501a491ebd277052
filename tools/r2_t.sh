# GPU parity tests (all), output under gpurun_out/r2t
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2t
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2t/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2t/pytest.log
