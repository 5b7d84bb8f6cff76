# ncu --set full of the dominant kernels of each config (summaries kept; .ncu-rep dropped: 64 MiB cap)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
CONFIG=rn50_mnv2 NCU_C=1 FOCUS="be:features.2.expand_bn.bwd_dx be:features.3.dw.wgrad be:features.2.expand.wgrad be:features.0.wgrad hp:layer2.2.conv2" bash tools/ncu_focus.sh
CONFIG=bert_rn50 NCU_C=1 FOCUS="hp:layer0.ffn2 hp:layer0.attn be:layer1.2.conv1.wgrad be:layer1.0.conv2.wgrad" bash tools/ncu_focus.sh
CONFIG=rn101_enc NCU_C=1 FOCUS="be:enc0.attn_bwd_dkv be:enc0.ln1.bwd" bash tools/ncu_focus.sh
for f in gpurun_out/ncu_*.ncu-rep; do python tools/ncu_report.py $f > ${f%.ncu-rep}.txt 2>&1; done
mkdir -p /tmp/ncurep; mv gpurun_out/*.ncu-rep /tmp/ncurep/ 2>/dev/null
du -sh gpurun_out
