cd "${GRAFT_REPO_ROOT:-.}"
python -m paper_conf_asplos_xiezggl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "freebase" --durations=5 > gpurun_out/r2_freebase.log 2>&1
python bench.py > gpurun_out/r2_bench_join.json 2> gpurun_out/r2_bench_join.err
bash tools/profile_round.sh criteo_kaggle
ls gpurun_out/prof_criteo_kaggle
