set -x
export MODES=0
ncu --set full --clock-control none --import-source on -k regex:gemm_tc_kernel -s 3 -c 1 -f -o gpurun_out/r1_gemm_pair_ffn1 python tools/gemm_one.py 16384 4096 1024 0 0 bf16 0.0 > gpurun_out/ncu1.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:gemm_tc_kernel -s 3 -c 1 -f -o gpurun_out/r1_gemm_pair_qkv python tools/gemm_one.py 16384 1024 1024 0 0 bf16 0.0 > gpurun_out/ncu2.log 2>&1
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bert.csv python tools/launch_list.py bert_large 0.25 graph > gpurun_out/ncu3.log 2>&1
ls -la gpurun_out/
