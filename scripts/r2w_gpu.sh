cd $GRAFT_REPO_ROOT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > /dev/null 2>&1
bash scripts/ab_gpu.sh r2w "c3 c2" "X=0" 2
