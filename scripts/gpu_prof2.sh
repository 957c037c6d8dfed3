mkdir -p gpurun_out
timeout 600 python scripts/prof_one.py X64_32768_256 fp32 1 > gpurun_out/prof2.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/prof_c2_fp64_v1 python scripts/prof_one.py C2 fp64 1 >> gpurun_out/prof2.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/prof_x64_fp32_v1 python scripts/prof_one.py X64_32768_256 fp32 1 >> gpurun_out/prof2.txt 2>&1
tail -5 gpurun_out/prof2.txt
