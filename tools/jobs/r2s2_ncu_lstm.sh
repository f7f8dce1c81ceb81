mkdir -p gpurun_out
python tools/run_workload.py cfg3_lstm_b64 3 --no-cublas && \
ncu --set full --clock-control none --import-source on -k regex:hgemm -s 2 -c 1 -o gpurun_out/s2_lstm64_relaxed python tools/run_workload.py cfg3_lstm_b64 3 --no-cublas > gpurun_out/s2_ncu5.log 2>&1
python tools/run_workload.py cfg3_bert_ffn2_4096 3 --no-cublas && \
ncu --set full --clock-control none --import-source on -k regex:hgemm -s 2 -c 1 -o gpurun_out/s2_ffn2_relaxed python tools/run_workload.py cfg3_bert_ffn2_4096 3 --no-cublas > gpurun_out/s2_ncu6.log 2>&1
ls -la gpurun_out/*.ncu-rep
