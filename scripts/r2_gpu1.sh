set -x
nvidia-smi -L
python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r2_gpu_tests.txt
python bench.py --steps 100 --warmup 5 > gpurun_out/r2_bench1.jsonl 2> gpurun_out/r2_bench1.err
python bench.py --gpus 2 --steps 50 --warmup 5 > gpurun_out/r2_bench2.jsonl 2> gpurun_out/r2_bench2.err
python bench_configs.py --configs c2,c5 --partitions 1,8 --sweeps 50 --c5-sweeps 10 > gpurun_out/r2_cfg.jsonl 2> gpurun_out/r2_cfg.err
tail -3 gpurun_out/r2_gpu_tests.txt
