# round-end bundle: profiles (bench, launch list, ncu full capture, NCCL launch list),
# then the GPU suite and smoke
bash scripts/profile_round.sh
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest.log
tail -3 gpurun_out/pytest.log
grep -E "^FAILED|^ERROR" gpurun_out/pytest.log | head -20
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -2 gpurun_out/smoke.log
