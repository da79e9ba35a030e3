python -c "import __graft_entry__ as g; g.build()"
CFG=${CFG:-small}
run() { timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=$1 --master-addr 127.0.0.1 --master-port $2 tests/xproc_worker.py --config $CFG --mode 1 --stress 1 --versions $3 --fanout $4 2>&1 | grep -E "stress:|XPROC_RESULT|torn" | tail -5; }
{
echo "=== direct, early notify (batched system-scope seals + pipelined install_direct), 3 consumers"
VIPER_EARLY_NOTIFY=1 run 4 29701 400 0
echo "=== scatter-allgather, early notify, 3 consumers"
VIPER_EARLY_NOTIFY=1 run 4 29702 400 2
echo "=== chain, early notify, 3 consumers"
VIPER_EARLY_NOTIFY=1 run 4 29703 400 1
echo "=== push, early notify, 3 consumers"
VIPER_EARLY_NOTIFY=1 run 4 29704 400 4
echo "=== NVLS kernel path (unicast emulation), early notify, 1 consumer"
VIPER_TEST_NVLS_UNICAST=1 VIPER_EARLY_NOTIFY=1 run 2 29705 400 3
echo "=== copy engine, 3 consumers"
run 4 29706 400 101
} > gpurun_out/r2_stress_$CFG.log 2>&1
