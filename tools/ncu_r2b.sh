# round-2 second-session captures: stem, LR power pass (conv5_x layer, 16k rows), res2 halo 3x3
cd "$GRAFT_REPO_ROOT"
make -j32 -s 2>&1 | tail -2
bash tools/ncu_one.sh stem "conv1_pool_kernel" 2
bash tools/ncu_one.sh lrdot 'lr_dot_kernel<\(int\)4, \(int\)2, \(int\)2>' 5 --images 20000
bash tools/ncu_one.sh res2halo 'conv_tc_kernel<\(int\)64, \(int\)7' 3
for f in stem lrdot res2halo; do python tools/ncu_digest.py gpurun_out/ncu_one/$f.raw.csv; done
