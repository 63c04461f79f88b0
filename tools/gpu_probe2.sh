mkdir -p gpurun_out
M="l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"
timeout 300 ncu --metrics $M --csv --log-file gpurun_out/calib_tma2.csv ./tools/ncu_calib_tma > gpurun_out/calib_tma2.log 2>&1
for p in 1 6 12; do BCF_TRACE=$p timeout 300 python tools/trace_pass.py > gpurun_out/trace_p$p.txt 2>&1; done
echo done
