for eng in ws1 ws2 gs8 tma8; do for pub in 0 1 2 3; do for pdl in 0 1; do
  echo -n "pub=$pub pdl=$pdl "; GR_COPY=$eng GR_TEST_PUB=$pub GR_PDL=$pdl timeout 60 ./tools/enginebench
done; done; done
