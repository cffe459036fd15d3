mkdir -p gpurun_out/trace
python scripts/trace_report.py --bytes-per-rank 1048576 --out gpurun_out/trace/allreduce_1MiB > /dev/null 2>gpurun_out/trace/err1.log
python scripts/trace_report.py --bytes-per-rank 8388608 --out gpurun_out/trace/allreduce_8MiB > /dev/null 2>gpurun_out/trace/err2.log
python scripts/trace_report.py --bytes-per-rank 268435456 --calls 4 --out gpurun_out/trace/allreduce_256MiB > /dev/null 2>gpurun_out/trace/err3.log
python scripts/trace_report.py --bytes-per-rank 16777216 --mode staged --out gpurun_out/trace/allreduce_staged_16MiB > /dev/null 2>gpurun_out/trace/err4.log
python scripts/trace_report.py --coll alltoall --bytes-per-rank 33554432 --out gpurun_out/trace/alltoall_32MiB > /dev/null 2>gpurun_out/trace/err5.log
