# Paper-shaped client sweep on the current code (7B, clients of 4 x 100 tokens, r8 q,v; N = 1..32): batched SAVE
# step, Menos on-demand mode, Alg.2 serving loop, Eq.2 vs Eq.3 memory.
timeout 1500 python tools/sweep_clients.py > gpurun_out/r2cd_sweep_clients.jsonl 2> gpurun_out/r2cd_sweep.err; echo "sweep rc=$?"; tail -3 gpurun_out/r2cd_sweep.err; cat gpurun_out/r2cd_sweep_clients.jsonl | head -c 3000
