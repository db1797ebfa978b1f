mkdir -p gpurun_out/sel; rm -f gpurun_out/sel/*
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/sel/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --config C2 --task-mb 1024 > /dev/null 2>&1
python scripts/ncu_summary.py launches gpurun_out/sel/launches.csv | head -8
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_select -s 2 -c 1 -o gpurun_out/sel/prof python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --config C2 --task-mb 1024 > /dev/null 2>&1
python scripts/ncu_summary.py report gpurun_out/sel/prof.ncu-rep --json gpurun_out/sel/ncu_full_k_select_C2.json 2>&1 | head -20
ncu -i gpurun_out/sel/prof.ncu-rep --page source --csv --print-source sass > gpurun_out/sel/sass.csv 2>/dev/null; gzip -f gpurun_out/sel/sass.csv; rm -f gpurun_out/sel/prof.ncu-rep
