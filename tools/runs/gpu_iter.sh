python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; echo TESTS $? >> gpurun_out/t.log
python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/b.log 2>&1
tail -3 gpurun_out/t.log; grep -o "\"recon\": {[^}]*}" gpurun_out/b.log; grep -o "\"value\": [0-9.]*, \"unit\": \"4K frames/s\", \"n_gpus\"[^,]*, \"steps\"[^,]*, \"warmup\"[^,]*, \"ms_per_step\": [0-9.]*" gpurun_out/b.log
ncu --set full --import-source on --clock-control none -k regex:${NCU_K:-k_recon_step} -s 20 -c 1 -o gpurun_out/${NCU_O:-prof} python bench.py --streams 16 --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu.log 2>&1
