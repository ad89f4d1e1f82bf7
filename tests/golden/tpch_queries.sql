-- TPC-H Q1, Q3, Q4, Q5, Q6, Q7 with validation parameters (BASELINE config 4; the paper
-- runs TPC-H, PAPER.md:305, :595).  Texts: SURVEY.md App. A.2, rewritten for the
-- stored representation ONLY as the DESIGN.md readings require:
--   O5  decimals are scale-2 integers: (1 - l_discount) -> (100 - l_discount),
--       (1 + l_tax) -> (100 + l_tax); 0.05..0.07 -> 5..7; quantity < 24 -> < 2400.
--       Results are therefore scaled integers (scale 2, 4 or 6).
--   O11 dates are int yyyymmdd and date arithmetic is folded:
--       date '1998-12-01' - interval '90' day = 19980902,
--       date '1994-01-01' + interval '1' year = 19950101,
--       date '1993-07-01' + interval '3' month = 19931001,
--       extract(year from l_shipdate) = l_shipdate / 10000.
--   avg(x) is reported as sum(x) and count(*) (O10: the average is a double
--   computed at finalisation).  Q1's avg_disc uses sum(l_discount).  Q1 also
--   reports SQLite's own avg(x) of the scale-2 integers (the tests divide by 100),
--   which pins the oracle's AVG columns.
--   LIMIT 10 of Q3 is dropped here so the whole pre-LIMIT group set is compared (O9).
-- Used by tests/test_oracle_sqlite.py (SQLite 3.45) to pin the oracle.
-- @tpch1
select l_returnflag, l_linestatus, sum(l_quantity), sum(l_extendedprice),
       sum(l_extendedprice*(100-l_discount)), sum(l_extendedprice*(100-l_discount)*(100+l_tax)),
       sum(l_discount), count(*), avg(l_quantity), avg(l_extendedprice), avg(l_discount)
  from lineitem where l_shipdate <= 19980902
 group by l_returnflag, l_linestatus order by l_returnflag, l_linestatus;
-- @tpch2
-- Q2 (SIZE 15, TYPE BRASS, REGION EUROPE).  Reading O35: s_name is reported as
-- s_suppkey (TPC-H's s_name = 'Supplier#' || lpad(s_suppkey, 9, '0') sorts the same),
-- the free-text columns s_address, s_phone, s_comment are not generated, and LIMIT
-- 100 is dropped so the whole ordered set is compared.
select s_acctbal, s_suppkey, n_name, p_partkey, p_mfgr
  from part, supplier, partsupp, nation, region
 where p_partkey = ps_partkey and s_suppkey = ps_suppkey and p_size = 15
   and p_type like '%BRASS' and s_nationkey = n_nationkey and n_regionkey = r_regionkey
   and r_name = 'EUROPE'
   and ps_supplycost = (select min(ps_supplycost) from partsupp, supplier, nation, region
                         where p_partkey = ps_partkey and s_suppkey = ps_suppkey
                           and s_nationkey = n_nationkey and n_regionkey = r_regionkey
                           and r_name = 'EUROPE')
 order by s_acctbal desc, n_name, s_suppkey, p_partkey;
-- @tpch3
select l_orderkey, o_orderdate, o_shippriority, sum(l_extendedprice*(100-l_discount)) as revenue
  from customer, orders, lineitem
 where c_mktsegment = 'BUILDING' and c_custkey = o_custkey and l_orderkey = o_orderkey
   and o_orderdate < 19950315 and l_shipdate > 19950315
 group by l_orderkey, o_orderdate, o_shippriority order by revenue desc, o_orderdate;
-- @tpch4
select o_orderpriority, count(*) as order_count from orders
 where o_orderdate >= 19930701 and o_orderdate < 19931001
   and exists (select * from lineitem where l_orderkey = o_orderkey and l_commitdate < l_receiptdate)
 group by o_orderpriority order by o_orderpriority;
-- @tpch5
select n_name, sum(l_extendedprice*(100-l_discount)) as revenue
  from customer, orders, lineitem, supplier, nation, region
 where c_custkey = o_custkey and l_orderkey = o_orderkey and l_suppkey = s_suppkey
   and c_nationkey = s_nationkey and s_nationkey = n_nationkey and n_regionkey = r_regionkey
   and r_name = 'ASIA' and o_orderdate >= 19940101 and o_orderdate < 19950101
 group by n_name order by revenue desc;
-- @tpch6
select sum(l_extendedprice*l_discount) as revenue, count(*) from lineitem
 where l_shipdate >= 19940101 and l_shipdate < 19950101
   and l_discount between 5 and 7 and l_quantity < 2400;
-- @tpch7
select n1.n_name as supp_nation, n2.n_name as cust_nation, l_shipdate / 10000 as l_year,
       sum(l_extendedprice*(100-l_discount)) as revenue
  from supplier, lineitem, orders, customer, nation n1, nation n2
 where s_suppkey = l_suppkey and o_orderkey = l_orderkey and c_custkey = o_custkey
   and s_nationkey = n1.n_nationkey and c_nationkey = n2.n_nationkey
   and ((n1.n_name = 'FRANCE' and n2.n_name = 'GERMANY') or (n1.n_name = 'GERMANY' and n2.n_name = 'FRANCE'))
   and l_shipdate between 19950101 and 19961231
 group by supp_nation, cust_nation, l_year order by supp_nation, cust_nation, l_year;
