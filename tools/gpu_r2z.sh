# ncu source-level capture of the alternating-group attention backward (cfg1 and cfg3 shapes)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 2 -c 2 -o gpurun_out/r2z_ws_cfg1 python tools/attn_time.py 14 512x16 32 32 1 > gpurun_out/r2z_ncu1.log 2>&1; echo "ncu cfg1 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 2 -c 2 -o gpurun_out/r2z_ws_cfg3 python tools/attn_time.py 14 2048x16 40 40 1 > gpurun_out/r2z_ncu3.log 2>&1; echo "ncu cfg3 rc=$?"
