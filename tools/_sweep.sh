L=paper_conf_ipps_andersonbdk11_b200/libcaqr.so
for ct in 124 200 247 296 400; do echo "C3 chain_target=$ct"; CAQR_CHAIN_TARGET=$ct python tools/ab_time.py $L --m 110592 --n 100 --reps 40 --rounds 1; done
for ct in 148 220 280 296 444; do echo "C4 chain_target=$ct"; CAQR_CHAIN_TARGET=$ct python tools/ab_time.py $L --reps 10 --rounds 1; done
