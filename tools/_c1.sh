L=paper_conf_ipps_andersonbdk11_b200/libcaqr.so
for ct in 0 8 16 4; do
  if [ $ct = 0 ]; then unset CAQR_CHAIN_TARGET; else export CAQR_CHAIN_TARGET=$ct; fi
  echo "stream chain_target=$ct"; python tools/ab_time.py $L --m 4096 --n 16 --reps 50 --rounds 1
done
unset CAQR_CHAIN_TARGET
echo "fused (skinny off)"; CAQR_SKINNY_MIN_M=100000000 python tools/ab_time.py $L --m 4096 --n 16 --reps 50 --rounds 1
for ct in 4 8 16; do echo "fused chain_target=$ct"; CAQR_CHAIN_TARGET=$ct CAQR_SKINNY_MIN_M=100000000 python tools/ab_time.py $L --m 4096 --n 16 --reps 50 --rounds 1; done
echo "C2 stream"; python tools/ab_time.py $L --m 4000000 --n 8 --reps 30 --rounds 1
echo "C2 fused"; CAQR_SKINNY_MIN_M=100000000 python tools/ab_time.py $L --m 4000000 --n 8 --reps 30 --rounds 1
