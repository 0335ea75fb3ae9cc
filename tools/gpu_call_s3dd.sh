ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:fop_ -c 7 -o gpurun_out/prof_r01_s3_variants python tools/profile_variants.py > gpurun_out/prof_variants.log 2>&1; echo ncu=$?
tail -9 gpurun_out/prof_variants.log
