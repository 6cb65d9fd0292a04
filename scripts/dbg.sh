cd $GRAFT_REPO_ROOT
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1
timeout 240 python -m pytest tests/test_gpu_brs.py -x -q --timeout 200 --durations=0 -p no:cacheprovider > gpurun_out/brs.log 2>&1; echo "brs rc=$?"; tail -25 gpurun_out/brs.log
timeout 200 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b1.log 2>&1; echo "bench rc=$?"; tail -2 gpurun_out/b1.log | cut -c1-300
