mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for C in google8 reddit; do
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 5 --warmup 3 --config $C --share-gpu > gpurun_out/multi2_$C.json 2> gpurun_out/multi2_$C.err; echo "multi2 $C rc=$?"; tail -c 1500 gpurun_out/multi2_$C.json; tail -3 gpurun_out/multi2_$C.err
done
for T in 1 0; do timeout 300 python bench.py --config tiny --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-torch-baseline --opt tma=$T | python3 -c "
import json,sys; d=json.loads(sys.stdin.read()); print('tiny tma=$T', d['ms_per_layer'])"; done
