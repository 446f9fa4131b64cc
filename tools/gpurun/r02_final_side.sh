# one gpurun call: the c2 bench line (BASELINE configs[1]) and the c3 sweep on the DNA pipeline with the final build
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 1200 python bench.py --workload c2 > gpurun_out/fs_c2.json 2> gpurun_out/fs_c2.err; echo c2=$?
timeout 1500 python tools/sweep_c3_dna.py > gpurun_out/fs_c3.txt 2> gpurun_out/fs_c3.err; echo c3=$?
