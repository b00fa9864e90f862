set -x
python tools/swap_profile.py resnet50 0.25 > gpurun_out/swap_resnet50.log 2>&1
python tools/swap_profile.py bert_large 0.25 6 > gpurun_out/swap_bert.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/hbm_step.csv python tools/step_once.py 2 0.25 > gpurun_out/hbm_step.log 2>&1
python tools/hbm_kernels.py gpurun_out/hbm_step.csv gpurun_out/r2_hbm_kernels.json > gpurun_out/hbm_summary.txt 2>&1
tail -3 gpurun_out/swap_resnet50.log gpurun_out/swap_bert.log gpurun_out/hbm_summary.txt
