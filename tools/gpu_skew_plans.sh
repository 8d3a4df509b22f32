# Plan arithmetic at 8-GPU BASELINE sizes (one GPU generates every rank's histograms)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/plans
python tools/skew_plan.py --workload zipf --z 1.0 > gpurun_out/plans/m4_z1.json; echo "m4 z1 rc=$?"
python tools/skew_plan.py --workload zipf --z 0.5 > gpurun_out/plans/m4_z05.json; echo "m4 z05 rc=$?"
python tools/skew_plan.py --workload unique --log2-r-per-gpu 29 --placement-z 1.0 > gpurun_out/plans/m2_placement_z1.json; echo "m2 pz1 rc=$?"
python tools/skew_plan.py --workload unique --log2-r-per-gpu 29 --placement-z 0.5 > gpurun_out/plans/m2_placement_z05.json; echo "m2 pz05 rc=$?"
python tools/skew_plan.py --workload zipf --z 1.0 --placement-z 1.0 > gpurun_out/plans/m4_z1_placement_z1.json; echo "m4 z1 pz1 rc=$?"
