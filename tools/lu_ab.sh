# L56 / GJ56 parity + timing (tools/lu_time.py) with the left-looking LU on and off
python -m pytest tests/test_gpu_lu.py -q -p no:cacheprovider 2>&1 | tail -3 > gpurun_out/pt_lu.txt
python bench.py --config L56 --no-also --no-c5 --no-cpu --steps 50 > gpurun_out/bench_l56.json 2> gpurun_out/bench_l56.err
