cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke=$?"
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_full.log 2>&1; echo "pytest=$?"
rm -f gpurun_out/sanitize_summary.txt
bash tools/sanitize.sh > /dev/null 2>&1; echo "sanitize done"
