# per-rank latency tables (FLUX, SD3; k virtual ranks serialised) + per-class SP breakdown at 2048^2
cd $GRAFT_REPO_ROOT
O=gpurun_out
mkdir -p $O
timeout -s KILL 1200 python tools/latency_table_model.py --serial --iters 5 --out $O/latency_table_serial.json > /dev/null 2> $O/ltm.err; echo "ltm $?"
timeout -s KILL 1200 python tools/latency_table_model.py --serial --model sd3 --iters 5 --out $O/latency_table_serial_sd3.json > /dev/null 2> $O/ltm_sd3.err; echo "ltm sd3 $?"
TSV_VIRTUAL_SERIAL=1 timeout -s KILL 900 python tools/sp_breakdown.py --res 1024,2048 --ks 1,2,4,8 --out $O/sp_breakdown.jsonl > /dev/null 2> $O/spb.err; echo "spb $?"
TSV_VIRTUAL_SERIAL=1 timeout -s KILL 900 python tools/sp_breakdown.py --model sd3 --res 1024,2048 --ks 1,2,4,8 --out $O/sp_breakdown_sd3.jsonl > /dev/null 2> $O/spb3.err; echo "spb sd3 $?"
