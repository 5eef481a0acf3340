mkdir -p gpurun_out
python tools/sweep.py --sizes 112,128,144,160,192,224,256 --dtypes f32 --steps 5 > gpurun_out/sw_f32.jsonl 2>&1
python tools/sweep.py --sizes 112,144,160 --dtypes c64 --steps 5 > gpurun_out/sw_c64.jsonl 2>&1
python tools/sweep.py --sizes 112 --dtypes c64 --steps 5 --variant alt_c64_R16G16_7x7_cta > gpurun_out/sw_alt1.jsonl 2>&1
python tools/sweep.py --sizes 144 --dtypes c64 --steps 5 --variant alt_c64_R16G16_9x9_cta > gpurun_out/sw_alt2.jsonl 2>&1
