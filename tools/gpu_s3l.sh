bash tools/round_profile.sh
bash tools/prof_full.sh s3l
ncu -i gpurun_out/prof_s3l.ncu-rep --page raw --csv > gpurun_out/prof_s3l_raw.csv 2>/dev/null
ls -la gpurun_out | tail -5
